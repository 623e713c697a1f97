"""tcgen05 kernel, TMA operand boxes vs cp.async producers: per TCCG case and dtype, the
planner's plan timed both ways (L2 flushed), GFLOP/s, fraction of the HBM roofline and of the
dtype's tensor peak.  Usage: python tools/umma_tma_bench.py [ids] [dtypes]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

HBM = 6547.8e9
PEAK = {"bf16": 1645e12, "tf32": 1645e12 / 2}
TDT = {"bf16": torch.bfloat16, "tf32": torch.float32}
ES = {"bf16": 2, "tf32": 4}
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


ids = ([int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 and sys.argv[1] != "all"
       else list(range(1, 49)))
dts = sys.argv[2].split(",") if len(sys.argv) > 2 else ["bf16", "tf32"]
for dt in dts:
    for c in [c for c in tcinputs.tccg48() if c.id in ids]:
        p = tc.plan(c.expr, c.extents, dtype=dt)
        A = tcinputs.uniform(p.numel("A"), 1000 + c.id, device="cuda").to(TDT[dt])
        B = tcinputs.uniform(p.numel("B"), 2000 + c.id, device="cuda").to(TDT[dt])
        C = torch.empty(p.numel("C"), dtype=TDT[dt], device="cuda")
        byts = ES[dt] * (p.numel("A") + p.numel("B") + p.numel("C"))
        row = {"id": c.id, "dtype": dt, "expr": c.expr, "tma": p.info()["tma_operands"], "pair": p.info()["cta_pair"],
               "variant": p.info()["variant"], "pred_ms": round(p.info()["t_pred_ms"], 4)}
        for name, kw in (("tma", {}), ("cpasync", {"tma_operands": False})):
            q = tc.plan(c.expr, c.extents, dtype=dt, **kw)
            ms = timeit(q, A, B, C)
            row[name] = {"ms": round(ms, 4), "tflops": round(q.flops / ms / 1e9, 1),
                         "hbm_frac": round(byts / (ms * 1e-3) / HBM, 3),
                         "peak_frac": round(q.flops / (ms * 1e-3) / PEAK[dt], 3)}
        print(json.dumps(row), flush=True)
        del A, B, C
