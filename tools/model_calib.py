"""Cost-model calibration data (planner.cpp model_time): for every TCCG-48 case in FP64, every
variant the B200 model ranked (stats.per_variant), the model's predicted time of that variant's
best configuration and its measured time (forced variant, L2 flushed, median of 3).
One JSON line per case: {"id", "rows": [[variant, pred_ms, measured_ms], ...]}."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402


def timeit(fn, flush, reps=3):
    ts = []
    for i in range(reps + 1):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        if i >= 1:
            ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]


flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ids = [int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 else list(range(1, 49))
for c in [c for c in tcinputs.tccg48() if c.id in ids]:
    p = tc.plan(c.expr, c.extents, "f64", stream=False)
    A = tcinputs.uniform(p.numel("A"), 1000 + c.id, device="cuda")
    B = tcinputs.uniform(p.numel("B"), 2000 + c.id, device="cuda")
    C = torch.empty(p.numel("C"), dtype=torch.float64, device="cuda")
    rows = []
    for v, _ in p.info()["stats"]["per_variant"]:
        pv = tc.plan(c.expr, c.extents, "f64", variant=v, stream=False)
        rows.append([v, round(pv.info()["t_pred_ms"], 5), round(timeit(lambda: pv.execute(A, B, C), flush), 5)])
    print(json.dumps({"id": c.id, "rows": rows}), flush=True)
