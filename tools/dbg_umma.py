"""UMMA ablation timings (development tool): dbg & 2 no MMA, & 4 no epilogue, & 8 no loads.
usage: python tools/dbg_umma.py <case> <dtype> [dbg,...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402
from tools.variant_sweep import time_plan  # noqa: E402

torch.cuda.set_device(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for spec in sys.argv[1:]:
    cid, dt = spec.split(":")
    case = [c for c in tcinputs.tccg48() if c.id == int(cid)][0]
    tdt = {"bf16": torch.bfloat16, "f32": torch.float32, "tf32": torch.float32}[dt]
    p0 = tc.plan(case.expr, case.extents, dtype=dt)
    A = tcinputs.uniform(p0.numel("A"), 1, device="cuda").to(tdt)
    B = tcinputs.uniform(p0.numel("B"), 2, device="cuda").to(tdt)
    C = torch.empty(p0.numel("C"), dtype=tdt, device="cuda")
    row = []
    for d in [int(x) for x in os.environ.get("DBGS", "0,2,4,8,6,12,14").split(",")]:
        p = tc.plan(case.expr, case.extents, dtype=dt, dbg=d)
        row.append(f"dbg{d}:{time_plan(p, A, B, C, flush):.4f}")
    i = p0.info()
    print(cid, dt, i["variant"], i["cs0"], i["Mt"], i["Nt"], i["Kt"], i["nsteps"], " ".join(row), flush=True)
