"""One libtc plan launched 3 times (for ncu captures).
usage: expr extents dtype [tiles|-] [variant|-] [tma_operands 0/1] [beta] [morder C/X]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

a = sys.argv[1:] + ["-"] * 7
expr, ext, dt, tiles, var, tma, beta, morder = a[:8]
tdt = {"bf16": torch.bfloat16, "f32": torch.float32, "tf32": torch.float32, "f64": torch.float64}[dt]
kw = {}
if tiles != "-":
    kw["force_tiles"] = tiles
if var != "-":
    kw["variant"] = int(var)
if tma != "-":
    kw["tma_operands"] = tma == "1"
b = 0.0 if beta == "-" else float(beta)
if morder != "-":
    kw["morder"] = morder
if os.environ.get("RUN_ONE_TMA_EPI") == "1":
    kw["tma"] = True
p = tc.plan(expr, ext, dtype=dt, **kw)
A = tcinputs.uniform(p.numel("A"), 1, device="cuda").to(tdt)
B = tcinputs.uniform(p.numel("B"), 2, device="cuda").to(tdt)
C = torch.zeros(p.numel("C"), dtype=tdt, device="cuda")
for _ in range(3):
    p.execute(A, B, C, beta=b)
torch.cuda.synchronize()
i = p.info()
print({k: i[k] for k in ("variant", "Mt", "Nt", "Kt", "nsteps", "nctas", "t_pred_ms", "m", "vecX", "wfX", "stg")})
