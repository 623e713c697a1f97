"""Ablation timing of the fused group kernel: side builds of libtc with -DTC_GROUP_ABLATE=k
(1: producers skip the gathers, 2: consumers skip the DMMAs, 3: consumers skip the flushes),
each timed on the triples group.  usage: python tools/group_ablation.py build | run EXTENTS"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def so(k):
    return os.path.join(ROOT, "paper_conf_cgo_kimstkpprs19_b200", "build", f"abl{k}", "libtc.so")


if sys.argv[1] == "build":
    from paper_conf_cgo_kimstkpprs19_b200 import build as b
    flags = list(b.NVCC_FLAGS)
    for k in (1, 2, 3):
        b.NVCC_FLAGS = flags + [f"-DTC_GROUP_ABLATE={k}"]
        b.SO = so(k)
        os.makedirs(os.path.dirname(b.SO), exist_ok=True)
        b.build(force=True)
elif sys.argv[1] == "run":
    ext = sys.argv[2]
    for k in (0, 1, 2, 3):
        env = dict(os.environ)
        if k:
            env["LIBTC_SO"] = so(k)
        out = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "bench_fused.py"), ext],
                             capture_output=True, text=True, env=env).stdout.strip().splitlines()
        row = json.loads(out[-1]) if out else {}
        print(json.dumps({"ablate": k, "fused_ms_b0": row.get("fused_ms_b0"), "fused_frac_b0": row.get("fused_frac_b0")}))
