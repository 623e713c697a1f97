"""ab-ac-cb (TCCG #18) BF16 at the BASELINE extents: forced tile shapes, TMA operand boxes vs
cp.async producers (development sweep; L2 flushed between launches)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timeit(p, A, B, C, reps=7):
    ts = []
    for i in range(reps + 2):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        p.execute(A, B, C)
        e1.record()
        e1.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]


expr = sys.argv[1] if len(sys.argv) > 1 else "ab-ac-cb"
ext = sys.argv[2] if len(sys.argv) > 2 else "a:5136;b:5120;c:5136"
dt = sys.argv[3] if len(sys.argv) > 3 else "bf16"
tdt = torch.bfloat16 if dt == "bf16" else torch.float32
tiles = sys.argv[4].split(",") if len(sys.argv) > 4 else [None, "a:128;b:128;c:64"]
p0 = tc.plan(expr, ext, dtype=dt)
A = tcinputs.uniform(p0.numel("A"), 1, device="cuda").to(tdt)
B = tcinputs.uniform(p0.numel("B"), 2, device="cuda").to(tdt)
C = torch.empty(p0.numel("C"), dtype=tdt, device="cuda")
for t in tiles:
    for name, kw in (("pair", {"pair": True}), ("tma", {"pair": False}), ("cpasync", {"tma_operands": False})):
        p = tc.plan(expr, ext, dtype=dt, force_tiles=t, **kw)
        ms = timeit(p, A, B, C)
        i = p.info()
        print(json.dumps({"tiles": t, "mode": name, "tma": i["tma_operands"], "pair": i["cta_pair"],
                          "ms": round(ms, 4), "tflops": round(p.flops / ms / 1e9, 1), "variant": i["variant"],
                          "Kt": i["Kt"], "pred_ms": round(i["t_pred_ms"], 4)}), flush=True)
