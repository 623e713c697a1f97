"""The streaming path forced on chosen TCCG cases (each of its three ranked configurations) vs the
tile kernel's model plan; L2 flushed, median of 5.  usage: python tools/stream_time.py <ids> [dtype]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402


def timeit(fn, flush, reps=5):
    ts = []
    for i in range(reps + 2):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]


flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ids = [int(x) for x in sys.argv[1].split(",")]
dt = sys.argv[2] if len(sys.argv) > 2 else "f64"
tdt = {"f64": torch.float64, "bf16": torch.bfloat16, "f32": torch.float32, "tf32": torch.float32}[dt]
for c in [c for c in tcinputs.tccg48() if c.id in ids]:
    pt = tc.plan(c.expr, c.extents, dt, stream=False)
    A = tcinputs.uniform(pt.numel("A"), 1000 + c.id, device="cuda").to(tdt)
    B = tcinputs.uniform(pt.numel("B"), 2000 + c.id, device="cuda").to(tdt)
    C = torch.empty(pt.numel("C"), dtype=tdt, device="cuda")
    row = {"id": c.id, "tile_ms": round(timeit(lambda: pt.execute(A, B, C), flush), 4)}
    for r in range(3):
        try:
            ps = tc.plan(c.expr, c.extents, dt, stream=True, stream_rank=r)
            s = ps.info()["stream"]
            row[f"stream{r}_ms"] = round(timeit(lambda: ps.execute(A, B, C), flush), 4)
            row[f"stream{r}"] = [s.get("tiles"), s.get("AR"), s.get("units"), s.get("KB"), s.get("stages")]
        except Exception as e:  # noqa: BLE001
            row[f"stream{r}"] = str(e)[:60]
    print(json.dumps(row), flush=True)
