"""Ablation timings (development tool): one TCCG case, one variant, kernel debug knobs
(dbg & 1: no C stores, & 2: no DMMA, & 4: no operand loads).
usage: python tools/dbg_exp.py <case> <variant,...> [dbg,...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402
from tools.variant_sweep import time_plan  # noqa: E402

cid = int(sys.argv[1])
vs = [int(x) for x in sys.argv[2].split(",")]
dbgs = [int(x) for x in sys.argv[3].split(",")] if len(sys.argv) > 3 else [0, 1, 2, 3, 4, 5, 6, 7]
case = [c for c in tcinputs.tccg48() if c.id == cid][0]
torch.cuda.set_device(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
p0 = tc.plan(case.expr, case.extents)
A = tcinputs.uniform(p0.numel("A"), 1, device="cuda")
B = tcinputs.uniform(p0.numel("B"), 2, device="cuda")
C = torch.empty(p0.numel("C"), dtype=torch.float64, device="cuda")
for v in vs:
    row = []
    for d in dbgs:
        p = tc.plan(case.expr, case.extents, variant=v, dbg=d)
        row.append(f"dbg{d}:{time_plan(p, A, B, C, flush):.4f}")
    print(cid, f"v{v}", " ".join(row), flush=True)
