"""Ablation of the tcgen05 kernel on the memory-bound BF16 / TF32 suite: side builds with
-DTC_UMMA_ABLATE=1 (epilogue drains nothing) and =2 (producers load nothing), timed against
the shipped library.  usage: python tools/umma_ablation.py build | run [ids] [dtypes]"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def so(k):
    return os.path.join(ROOT, "paper_conf_cgo_kimstkpprs19_b200", "build", f"uabl{k}", "libtc.so")


if sys.argv[1] == "build":
    from paper_conf_cgo_kimstkpprs19_b200 import build as b
    flags = list(b.NVCC_FLAGS)
    for k in (1, 2):
        b.NVCC_FLAGS = flags + [f"-DTC_UMMA_ABLATE={k}"]
        b.SO = so(k)
        os.makedirs(os.path.dirname(b.SO), exist_ok=True)
        b.build(force=True)
else:
    for k in (0, 1, 2):
        env = dict(os.environ)
        if k:
            env["LIBTC_SO"] = so(k)
        print("== ablate", k, flush=True)
        subprocess.run([sys.executable, os.path.join(ROOT, "tools", "umma_tma_bench.py")] + sys.argv[2:], env=env)
