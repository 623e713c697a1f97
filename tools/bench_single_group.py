"""Single CCSD(T) contractions (TCCG #31-48) through the fused group kernel (a group of one)
vs tc_execute (tuned plan), at beta 0 and 1; one JSON line per case."""
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
ids = [int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 else list(range(31, 49))
for c in [c for c in tcinputs.tccg48() if c.id in ids]:
    p = tc.plan(c.expr, c.extents)
    A = tcinputs.uniform(p.numel("A"), 1000 + c.id, device="cuda")
    B = tcinputs.uniform(p.numel("B"), 2000 + c.id, device="cuda")
    C = torch.zeros(p.numel("C"), dtype=torch.float64, device="cuda")
    g = tc.plan_group([p])
    row = {"id": c.id, "tile": g.info()["T"], "tma": g.info()["tma"]}
    for beta in (0.0, 1.0):
        pt = p.tuned(A, B, C, topk=8, reps=2, beta=beta)
        row[f"plan_b{int(beta)}_ms"] = round(timeit(lambda: pt.execute(A, B, C, beta=beta), flush), 4)
        row[f"group_b{int(beta)}_ms"] = round(timeit(lambda: g.execute([A], [B], C, 1.0, beta), flush), 4)
    print(json.dumps(row), flush=True)
