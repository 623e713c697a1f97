"""Forced FP64 variants against the tuned plan on chosen TCCG cases (L2 flushed, median of 5).
usage: python tools/variant_ab.py <ids> <variants>"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402


def timeit(fn, flush, reps=5):
    ts = []
    for i in range(reps + 2):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]


flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ids = [int(x) for x in sys.argv[1].split(",")]
vs = [int(x) for x in sys.argv[2].split(",")]
for c in [c for c in tcinputs.tccg48() if c.id in ids]:
    p = tc.plan(c.expr, c.extents, "f64")
    A = tcinputs.uniform(p.numel("A"), 1000 + c.id, device="cuda")
    B = tcinputs.uniform(p.numel("B"), 2000 + c.id, device="cuda")
    C = torch.empty(p.numel("C"), dtype=torch.float64, device="cuda")
    t = p.tuned(A, B, C, topk=8, reps=2)
    row = {"id": c.id, "tuned_v": t.info()["variant"], "tuned_ms": round(timeit(lambda: t.execute(A, B, C), flush), 4),
           "model_v": p.info()["variant"]}
    for v in vs:
        try:
            pv = tc.plan(c.expr, c.extents, "f64", variant=v)
            row[f"v{v}"] = round(timeit(lambda: pv.execute(A, B, C), flush), 4)
        except Exception as e:  # noqa: BLE001
            row[f"v{v}"] = str(e)[:40]
    print(json.dumps(row), flush=True)
