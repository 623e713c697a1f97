"""One FP64 launch of TCCG #31 (sd_t_d1 abcdef-dega-gfbc) with beta = 0, then beta = 1, for
an ncu capture of what reading C (beta != 0) costs the direct epilogue."""
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

torch.cuda.set_device(0)
c = [x for x in tcinputs.tccg48() if x.id == 31][0]
p = tc.plan(c.expr, c.extents)
A = torch.rand(p.numel("A"), dtype=torch.float64, device="cuda")
B = torch.rand(p.numel("B"), dtype=torch.float64, device="cuda")
C = torch.rand(p.numel("C"), dtype=torch.float64, device="cuda")
for beta in (0.0, 1.0):
    p.execute(A, B, C, 1.0, beta)
torch.cuda.synchronize()
print("variant", p.info()["variant"])
