"""One fused triples group launch pattern for ncu: python tools/run_fused.py EXTENTS [reps]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

ext = sys.argv[1] if len(sys.argv) > 1 else ";".join(f"{x}:24" for x in "abcdefg")
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
exprs = [c.expr for c in tcinputs.tccg48() if c.group.startswith("CCSDT")]
plans = [tc.plan(e, ext) for e in exprs]
A = [tcinputs.uniform(p.numel("A"), 1000 + i, device="cuda") for i, p in enumerate(plans)]
B = [tcinputs.uniform(p.numel("B"), 2000 + i, device="cuda") for i, p in enumerate(plans)]
C = torch.empty(plans[0].numel("C"), dtype=torch.float64, device="cuda")
g = tc.plan_group(plans)
for _ in range(reps):
    g.execute(A, B, C)
torch.cuda.synchronize()
print(g.info()["T"], g.info()["grid"])
