"""Run one UMMA case with a dbg value a few times (ncu target).  usage: dbg_one.py case dtype dbg"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402
cid, dt, dbg = int(sys.argv[1]), sys.argv[2], int(sys.argv[3])
case = [c for c in tcinputs.tccg48() if c.id == cid][0]
tdt = {"bf16": torch.bfloat16, "f32": torch.float32, "tf32": torch.float32}[dt]
p = tc.plan(case.expr, case.extents, dtype=dt, dbg=dbg)
A = tcinputs.uniform(p.numel("A"), 1, device="cuda").to(tdt)
B = tcinputs.uniform(p.numel("B"), 2, device="cuda").to(tdt)
C = torch.empty(p.numel("C"), dtype=tdt, device="cuda")
for _ in range(3):
    p.execute(A, B, C)
torch.cuda.synchronize()
