"""Hand-off timeline of the fused group kernel (CTA 0): builds a -DTC_GROUP_TRACE libtc on the
side and prints per-step clock deltas.  usage: python tools/group_trace.py build | run EXTENTS"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
SO = os.path.join(ROOT, "paper_conf_cgo_kimstkpprs19_b200", "build", "trace_group", "libtc.so")
if sys.argv[1] == "build":
    from paper_conf_cgo_kimstkpprs19_b200 import build as b
    b.NVCC_FLAGS = b.NVCC_FLAGS + ["-DTC_GROUP_TRACE"]
    b.SO = SO
    os.makedirs(os.path.dirname(SO), exist_ok=True)
    b.build(force=True)
    sys.exit(0)
os.environ["LIBTC_SO"] = SO
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

ext = sys.argv[2]
exprs = [c.expr for c in tcinputs.tccg48() if c.group.startswith("CCSDT")]
plans = [tc.plan(e, ext) for e in exprs]
A = [tcinputs.uniform(p.numel("A"), 1000 + i, device="cuda") for i, p in enumerate(plans)]
B = [tcinputs.uniform(p.numel("B"), 2000 + i, device="cuda") for i, p in enumerate(plans)]
C = torch.empty(plans[0].numel("C"), dtype=torch.float64, device="cuda")
g = tc.plan_group(plans)
tr = torch.zeros(8 * 1024, dtype=torch.int64, device="cuda")
os.environ["TC_GROUP_TRACE_PTR"] = str(tr.data_ptr())
for _ in range(3):
    tr.zero_()
    g.execute(A, B, C)
torch.cuda.synchronize()
t = tr.view(8, 1024).cpu().numpy().astype("int64")
names = {0: "c_full", 1: "c_mma_done", 6: "c_flush_bar", 2: "c_flush_done", 3: "p_top", 4: "p_empty", 5: "p_issued"}
t0 = t[t > 0].min()
print("step " + " ".join(f"{names[k]:>12s}" for k in (3, 4, 5, 0, 1, 6, 2)))
for j in list(range(0, 40)) + list(range(200, 220)):
    print(f"{j:4d} " + " ".join(f"{(t[k, j] - t0) if t[k, j] else -1:12d}" for k in (3, 4, 5, 0, 1, 6, 2)))
import numpy as np  # noqa: E402
for a, b in ((0, 1), (1, 6), (6, 2), (3, 4), (4, 5), (5, 0)):
    d = [t[b, j] - t[a, j] for j in range(20, 500) if t[a, j] and t[b, j]]
    if d:
        print(f"{names[a]} -> {names[b]}: median {np.median(d):.0f} clk")
d = [t[0, j + 1] - t[0, j] for j in range(20, 500) if t[0, j] and t[0, j + 1]]
print(f"step period (consumer full->full): median {np.median(d):.0f} clk")
