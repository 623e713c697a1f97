"""Ablation of the streaming BF16 kernel (kernel_stream.cuh) on TCCG #1-8: side builds with
-DTC_STREAM_ABLATE=1 (no MMAs), 2 (no C stores), 3 (neither: the TMA X stream alone) and
-DTC_STREAM_PROMO=3 (X boxes with 256-B L2 promotion), timed against the shipped library.
usage: python tools/stream_ablation.py build | run [ids]"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
VARIANTS = {"abl1": ["-DTC_STREAM_ABLATE=1"], "abl2": ["-DTC_STREAM_ABLATE=2"], "abl3": ["-DTC_STREAM_ABLATE=3"],
            "promo256": ["-DTC_STREAM_PROMO=3"]}


def so(k):
    return os.path.join(ROOT, "paper_conf_cgo_kimstkpprs19_b200", "build", f"s{k}", "libtc.so")


if sys.argv[1] == "build":
    from paper_conf_cgo_kimstkpprs19_b200 import build as b
    flags = list(b.NVCC_FLAGS)
    for k, f in VARIANTS.items():
        b.NVCC_FLAGS = flags + f
        b.SO = so(k)
        os.makedirs(os.path.dirname(b.SO), exist_ok=True)
        b.build(force=True)
else:
    for k in ["base"] + list(VARIANTS):
        env = dict(os.environ)
        if k != "base":
            env["LIBTC_SO"] = so(k)
        print("== variant", k, flush=True)
        subprocess.run([sys.executable, os.path.join(ROOT, "tools", "stream_check.py")] + sys.argv[2:], env=env)
