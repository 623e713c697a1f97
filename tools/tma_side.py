"""Side builds of libtc for the tcgen05 TMA-operand experiments (L2 cache policy of the boxes,
L2 promotion of the maps) and a runner of tools/tma_sweep.py against each.
usage: python tools/tma_side.py build | run [sweep args...]"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
SIDES = {"pol0": ["-DTC_UMMA_TMA_POL=0"], "pol2": ["-DTC_UMMA_TMA_POL=2"],
         "promo0": ["-DTC_UMMA_TMA_PROMO=0"], "promo128": ["-DTC_UMMA_TMA_PROMO=2"]}


def so(k):
    return os.path.join(ROOT, "paper_conf_cgo_kimstkpprs19_b200", "build", f"side_{k}", "libtc.so")


if sys.argv[1] == "build":
    from paper_conf_cgo_kimstkpprs19_b200 import build as b
    flags = list(b.NVCC_FLAGS)
    for k, f in SIDES.items():
        b.NVCC_FLAGS = flags + f
        b.SO = so(k)
        os.makedirs(os.path.dirname(b.SO), exist_ok=True)
        b.build(force=True)
else:
    for k in ["default"] + list(SIDES):
        env = dict(os.environ)
        if k != "default":
            env["LIBTC_SO"] = so(k)
        print("==", k, flush=True)
        subprocess.run([sys.executable, os.path.join(ROOT, "tools", "tma_sweep.py")] + sys.argv[2:], env=env)
