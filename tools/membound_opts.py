"""FP64 memory-bound TCCG #1-8: measured time of the tuned plan under planner options (default;
m digits in X order; + TMA C-store epilogue), against the HBM roofline."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

HBM = 6547.8e9
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timeit(p, A, B, C, reps=5):
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


ids = [int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 else list(range(1, 9))
for c in [c for c in tcinputs.tccg48() if c.id in ids]:
    row = {"id": c.id}
    p0 = tc.plan(c.expr, c.extents)
    A = tcinputs.uniform(p0.numel("A"), 1000 + c.id, device="cuda")
    B = tcinputs.uniform(p0.numel("B"), 2000 + c.id, device="cuda")
    C = torch.empty(p0.numel("C"), dtype=torch.float64, device="cuda")
    byts = 8 * (p0.numel("A") + p0.numel("B") + p0.numel("C"))
    for name, kw in (("default", {}), ("morderX", {"morder": "X"}), ("tma", {"tma": True}),
                     ("morderX_tma", {"morder": "X", "tma": True})):
        try:
            p = tc.plan(c.expr, c.extents, **kw).tuned(A, B, C, topk=8, reps=2)
            ms = timeit(p, A, B, C)
            row[name] = {"ms": round(ms, 4), "hbm_frac": round(byts / (ms * 1e-3) / HBM, 3), "v": p.info()["variant"]}
        except Exception as e:  # noqa: BLE001
            row[name] = str(e)[:80]
    print(json.dumps(row), flush=True)
