"""FP64 tile-kernel epilogue store experiments on the near-ridge CCSD(T) cases (#31-48, C write
~ DMMA time) plus compute- and memory-bound checks: side builds with another store op
(-DTC_F64_ST_OP=...) timed against the shipped library, per FP64 variant, L2 flushed.
usage: python tools/f64_epi_ab.py build | run [ids]"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
VARIANTS = {"cs": ['-DTC_F64_ST_OP="st.global.cs.f64"'], "wt": ['-DTC_F64_ST_OP="st.global.wt.f64"']}
VLIST = [None, 0, 3, 4, 5, 10, 25]


def so(k):
    return os.path.join(ROOT, "paper_conf_cgo_kimstkpprs19_b200", "build", f"e{k}", "libtc.so")


def run(ids):
    import torch
    import tcinputs
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")

    def timeit(p, A, B, C, reps=7):
        ts = []
        for i in range(reps + 2):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            p.execute(A, B, C)
            e1.record()
            e1.synchronize()
            if i >= 2:
                ts.append(e0.elapsed_time(e1))
        return sorted(ts)[len(ts) // 2]

    for c in [c for c in tcinputs.tccg48() if c.id in ids]:
        p0 = tc.plan(c.expr, c.extents, stream=False)
        A = tcinputs.uniform(p0.numel("A"), 1, device="cuda")
        B = tcinputs.uniform(p0.numel("B"), 2, device="cuda")
        C = torch.zeros(p0.numel("C"), dtype=torch.float64, device="cuda")
        row = {"lib": (os.environ.get("LIBTC_SO") or "base/x").split("/")[-2], "id": c.id, "model_v": p0.info()["variant"]}
        for v in VLIST:
            try:
                p = tc.plan(c.expr, c.extents, variant=v, stream=False)
                row[f"v{v}"] = round(timeit(p, A, B, C) * 1e3, 1)
            except Exception:
                pass
        print(json.dumps(row), flush=True)


if sys.argv[1] == "build":
    from paper_conf_cgo_kimstkpprs19_b200 import build as b
    flags = list(b.NVCC_FLAGS)
    for k, f in VARIANTS.items():
        b.NVCC_FLAGS = flags + f
        b.SO = so(k)
        os.makedirs(os.path.dirname(b.SO), exist_ok=True)
        b.build(force=True)
elif sys.argv[1] == "one":
    run([int(x) for x in sys.argv[2].split(",")])
else:
    ids = sys.argv[2] if len(sys.argv) > 2 else "31,33,40,45,12,14,16,6,8,19"
    for k in ["base"] + list(VARIANTS):
        env = dict(os.environ)
        if k != "base":
            env["LIBTC_SO"] = so(k)
        subprocess.run([sys.executable, os.path.abspath(__file__), "one", ids], env=env)
