"""TCCG #31 (sd_t_d1) FP64, beta = 0 and beta = 1, for the planner's choice and every FP64
variant forced: which epilogue (direct / staged-deferred) pays least for reading C."""
import json
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200.csrc_variants import F64_VARIANTS, STG_VARIANTS  # noqa: E402

torch.cuda.set_device(0)
c = [x for x in tcinputs.tccg48() if x.id == 31][0]


def t(p, A, B, C, beta, reps=10):
    p.execute(A, B, C, 1.0, beta)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        p.execute(A, B, C, 1.0, beta)
    e1.record()
    torch.cuda.synchronize()
    return round(e0.elapsed_time(e1) / reps, 4)


for v in [None] + list(F64_VARIANTS):
    try:
        p = tc.plan(c.expr, c.extents, variant=v)
    except Exception as e:  # variant illegal for this case
        print(json.dumps({"variant": v, "error": str(e)[:80]}))
        continue
    A = torch.rand(p.numel("A"), dtype=torch.float64, device="cuda")
    B = torch.rand(p.numel("B"), dtype=torch.float64, device="cuda")
    C = torch.rand(p.numel("C"), dtype=torch.float64, device="cuda")
    vv = p.info()["variant"]
    print(json.dumps({"variant": v, "chosen": vv, "stg": vv in STG_VARIANTS, "beta0_ms": t(p, A, B, C, 0.0),
                      "beta1_ms": t(p, A, B, C, 1.0)}), flush=True)
