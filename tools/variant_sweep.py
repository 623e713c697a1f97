"""For selected TCCG cases, time the planner's best config within EVERY kernel variant and
print measured vs predicted time (calibration data for the B200 cost model).
usage: python tools/variant_sweep.py 1,3,9,12,31,40"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200.csrc_variants import F64_VARIANTS  # noqa: E402


def time_plan(p, A, B, C, flush, reps=5):
    for _ in range(2):
        p.execute(A, B, C)
    ts = []
    for _ in range(reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        p.execute(A, B, C)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    ids = [int(x) for x in sys.argv[1].split(",")]
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for case in tcinputs.tccg48():
        if case.id not in ids:
            continue
        p0 = tc.plan(case.expr, case.extents)
        A = tcinputs.uniform(p0.numel("A"), 1000 + case.id, device="cuda")
        B = tcinputs.uniform(p0.numel("B"), 2000 + case.id, device="cuda")
        C = torch.empty(p0.numel("C"), dtype=torch.float64, device="cuda")
        best = p0.info()["variant"]
        vs = [int(x) for x in os.environ["TC_VARIANTS"].split(",")] if os.environ.get("TC_VARIANTS") else F64_VARIANTS
        tmas = (False, True) if os.environ.get("TC_SWEEP_TMA") else (False,)
        for v, tma in [(v, t) for v in vs for t in tmas]:
            try:
                p = tc.plan(case.expr, case.extents, variant=v, tma=tma)
            except tc.TcError as e:
                print(json.dumps({"id": case.id, "variant": v, "error": str(e)}))
                continue
            i = p.info()
            ms = time_plan(p, A, B, C, flush)
            print(json.dumps({"id": case.id, "variant": v, "tma": tma, "chosen": v == best, "ms": round(ms, 4),
                              "pred_ms": round(i["t_pred_ms"], 4), "comp": round(i["t_comp_ms"], 4),
                              "mem": round(i["t_mem_ms"], 4), "l2": round(i["t_l2_ms"], 4),
                              "gflops": round(p.flops / ms / 1e6, 1), "Mt": i["Mt"], "Nt": i["Nt"],
                              "Kt": i["Kt"], "mo": i["morder"], "ko": i["korder"],
                              "wf": [i["wfX"], i["wfY"]], "vec": [i["vecX"], i["vecY"]],
                              "tiles": {x["name"]: x["tile"] for x in i["indices"]}}), flush=True)
        del A, B, C


if __name__ == "__main__":
    main()
