"""Time the fused CCSD(T) triples group (tc_group_execute) against the unfused group
(tc_execute_group, 18 launches) at several extents; one JSON line per extent."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

FP64_PEAK = 37.16e12
HBM = 6547.8e9


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


def main():
    exprs = [c.expr for c in tcinputs.tccg48() if c.group.startswith("CCSDT")]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    exts = sys.argv[1:] or ["a:24;b:16;c:16;d:24;e:16;f:16;g:24",
                            ";".join(f"{x}:16" for x in "abcdefg"), ";".join(f"{x}:24" for x in "abcdefg")]
    for ext in exts:
        plans = [tc.plan(e, ext) for e in exprs]
        A = [tcinputs.uniform(p.numel("A"), 1000 + i, device="cuda") for i, p in enumerate(plans)]
        B = [tcinputs.uniform(p.numel("B"), 2000 + i, device="cuda") for i, p in enumerate(plans)]
        C = torch.empty(plans[0].numel("C"), dtype=torch.float64, device="cuda")
        g = tc.plan_group(plans)
        flops = sum(p.flops for p in plans)
        byts = 8 * (sum(p.numel("A") + p.numel("B") for p in plans) + C.numel())
        attain = min(FP64_PEAK, flops / byts * HBM)
        row = {"extents": ext, "group": g.info()["T"], "BK": g.info()["BK"], "tma": g.info()["tma"]}
        for beta in (0.0, 1.0):
            ms = timeit(lambda: g.execute(A, B, C, 1.0, beta), flush)
            row[f"fused_ms_b{int(beta)}"] = round(ms, 4)
            row[f"fused_tflops_b{int(beta)}"] = round(flops / ms / 1e9, 3)
            row[f"fused_frac_b{int(beta)}"] = round(flops / (ms * 1e-3) / attain, 4)
        ms = timeit(lambda: tc.execute_group(plans, A, B, C), flush, reps=3)
        row["unfused_ms"] = round(ms, 4)
        row["unfused_tflops"] = round(flops / ms / 1e9, 3)
        print(json.dumps(row), flush=True)
        del A, B, C, plans, g
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
