"""Near-ridge CCSD(T) TCCG #31-48 (K = 24, FP64): time per FP64 variant with / without the
TMA C-store epilogue, at beta 0 and 1 (L2 flushed).  usage: python tools/ridge_opts.py [ids]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200.csrc_variants import F64_VARIANTS  # noqa: E402

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timeit(p, A, B, C, beta, reps=5):
    ts = []
    for i in range(reps + 2):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        p.execute(A, B, C, beta=beta)
        e1.record()
        e1.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]


ids = [int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 else [31, 33, 40]
for c in [c for c in tcinputs.tccg48() if c.id in ids]:
    p0 = tc.plan(c.expr, c.extents)
    A = tcinputs.uniform(p0.numel("A"), 1, device="cuda")
    B = tcinputs.uniform(p0.numel("B"), 2, device="cuda")
    C = torch.zeros(p0.numel("C"), dtype=torch.float64, device="cuda")
    row = {"id": c.id, "model_v": p0.info()["variant"]}
    for v in [None] + list(F64_VARIANTS):
        for tma in (False, True):
            for beta in (0.0, 1.0):
                try:
                    p = tc.plan(c.expr, c.extents, variant=v, tma=tma)
                    row[f"v{v}{'t' if tma else ''}b{int(beta)}"] = round(timeit(p, A, B, C, beta) * 1e3, 1)
                except Exception as e:
                    pass
    print(json.dumps(row), flush=True)
