"""One tcgen05 plan, launched 3 times (for ncu captures).  usage: expr extents dtype tiles tma(0/1)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

expr, ext, dt, tiles, tma = sys.argv[1:6]
tdt = torch.bfloat16 if dt == "bf16" else torch.float32
p = tc.plan(expr, ext, dtype=dt, force_tiles=None if tiles == "-" else tiles, tma_operands=tma == "1")
A = tcinputs.uniform(p.numel("A"), 1, device="cuda").to(tdt)
B = tcinputs.uniform(p.numel("B"), 2, device="cuda").to(tdt)
C = torch.empty(p.numel("C"), dtype=tdt, device="cuda")
for _ in range(3):
    p.execute(A, B, C)
torch.cuda.synchronize()
print(p.info()["tma_operands"])
