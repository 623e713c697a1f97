"""Per-case timing of the TCCG-48 suite (development tool; bench.py is the contract)."""
import json
import sys
import os

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402


def main():
    cost = sys.argv[1] if len(sys.argv) > 1 else "b200"
    dtype = os.environ.get("TC_DTYPE", "f64")
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float64
    ids = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else None
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    out = []
    for case in tcinputs.tccg48():
        if ids and case.id not in ids:
            continue
        p = tc.plan(case.expr, case.extents, cost=cost, dtype=dtype)
        info = p.info()
        A = tcinputs.uniform(p.numel("A"), 1000 + case.id, device="cuda").to(tdt)
        B = tcinputs.uniform(p.numel("B"), 2000 + case.id, device="cuda").to(tdt)
        C = torch.empty(p.numel("C"), dtype=tdt, device="cuda")
        for _ in range(3):
            p.execute(A, B, C)
        ts = []
        for _ in range(10):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            p.execute(A, B, C)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        ts.sort()
        ms = ts[len(ts) // 2]
        gf = p.flops / ms / 1e6
        r = {"id": case.id, "expr": case.expr, "ms": round(ms, 4), "gflops": round(gf, 1),
             "vec": [info["vecX"], info["vecY"]], "kmaj": [info["xKmajor"], info["yKmajor"]],
             "pred_ms": round(info["t_pred_ms"], 4), "variant": info["variant"],
             "Mt": info["Mt"], "Nt": info["Nt"], "Kt": info["Kt"],
             "tiles": {x["name"]: x["tile"] for x in info["indices"]}}
        out.append(r)
        print(json.dumps(r), flush=True)
        del A, B, C
    import math
    g = math.exp(sum(math.log(r["gflops"]) for r in out) / len(out))
    print(json.dumps({"geomean_gflops": round(g, 1), "n": len(out)}))


if __name__ == "__main__":
    main()
