"""The streaming BF16 path (stream.hpp) against the tcgen05 path on the memory-bound TCCG
cases #1-8 (and ragged variants): agreement of the two results and the time of each.
One JSON line per case."""
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
cases = [(c.id, c.expr, c.extents) for c in tcinputs.tccg48() if c.id <= 8]
cases += [(101, "abcde-efbad-cf", "a:20;b:3;c:13;d:5;e:44;f:9"),
          (102, "abc-bda-dc", "a:37;b:24;c:7;d:300"),
          (103, "abc-dca-bd", "a:40;b:17;c:3;d:33"),
          (104, "abcd-ebad-ce", "a:24;b:5;c:31;d:3;e:17")]
hbm = 6548.8
DT = sys.argv[2] if len(sys.argv) > 2 else "bf16"
TDT = {"bf16": torch.bfloat16, "f64": torch.float64, "f32": torch.float32, "tf32": torch.float32}[DT]
ES = {"bf16": 2, "f64": 8, "f32": 4, "tf32": 4}[DT]
if len(sys.argv) > 1 and sys.argv[1] != "all":
    keep = {int(x) for x in sys.argv[1].split(",")}
    cases = [c for c in cases if c[0] in keep]
for cid, expr, ext in cases:
    ps = tc.plan(expr, ext, DT, stream=True)
    pg = tc.plan(expr, ext, DT, stream=False)
    info = ps.info()["stream"]
    A = tcinputs.uniform(ps.numel("A"), 1000 + cid, device="cuda").to(TDT)
    B = tcinputs.uniform(ps.numel("B"), 2000 + cid, device="cuda").to(TDT)
    Cs = torch.full((ps.numel("C"),), float("nan"), dtype=TDT, device="cuda")
    Cg = torch.full((ps.numel("C"),), float("nan"), dtype=TDT, device="cuda")
    row = {"id": cid, "expr": expr, "stream": info}
    try:
        ps.execute(A, B, Cs)
        pg.execute(A, B, Cg)
        torch.cuda.synchronize()
        d = (Cs.double() - Cg.double()).abs()
        row["nan"] = int(torch.isnan(Cs.float()).sum())
        row["maxdiff"] = float(d.max())
        row["maxabs"] = float(Cg.float().abs().max())
        if cid <= 8:
            row["stream_ms"] = round(timeit(lambda: ps.execute(A, B, Cs), flush), 4)
            row["tcgen05_ms"] = round(timeit(lambda: pg.execute(A, B, Cg), flush), 4)
            by = ES * (ps.numel("A") + ps.numel("B") + ps.numel("C"))
            row["stream_hbm_frac"] = round(by / (row["stream_ms"] * 1e-3) / 1e9 / hbm, 4)
            row["tcgen05_hbm_frac"] = round(by / (row["tcgen05_ms"] * 1e-3) / 1e9 / hbm, 4)
    except Exception as e:  # noqa: BLE001
        row["error"] = repr(e)
    print(json.dumps(row), flush=True)
