"""Run one TCCG case a few times (target for ncu captures).
usage: python tools/run_case.py <id> [reps] [cost] [variant]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

cid = int(sys.argv[1])
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
cost = sys.argv[3] if len(sys.argv) > 3 else "b200"
variant = int(sys.argv[4]) if len(sys.argv) > 4 else None
case = [c for c in tcinputs.tccg48() if c.id == cid][0] if cid > 0 else tcinputs.eq1()
dtype = os.environ.get("TC_DTYPE", "f64")
tdt = {"bf16": torch.bfloat16, "f32": torch.float32, "tf32": torch.float32}.get(dtype, torch.float64)
p = tc.plan(case.expr, case.extents, cost=cost, variant=variant, dtype=dtype)
A = tcinputs.uniform(p.numel("A"), 1000 + cid, device="cuda").to(tdt)
B = tcinputs.uniform(p.numel("B"), 2000 + cid, device="cuda").to(tdt)
C = torch.empty(p.numel("C"), dtype=tdt, device="cuda")
for _ in range(reps):
    p.execute(A, B, C)
torch.cuda.synchronize()
print(case.id, case.expr, p.info()["variant"], p.info()["Mt"], p.info()["Nt"], p.info()["Kt"])
