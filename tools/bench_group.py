"""Time tc_execute_group on the 18 CCSD(T) triples (TCCG-48 cases 31-48 accumulated into one
t3, SURVEY 8(f) NEXT-4 first step), FP64, eager vs one CUDA graph, CUDA events on the
launching stream.  Prints one JSON line per extent set."""
import json
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402


def run(ext, reps=20):
    exprs = [c.expr for c in tcinputs.tccg48() if c.group.startswith("CCSDT")]
    plans = [tc.plan(e, ext) for e in exprs]
    A = [torch.rand(p.numel("A"), dtype=torch.float64, device="cuda") for p in plans]
    B = [torch.rand(p.numel("B"), dtype=torch.float64, device="cuda") for p in plans]
    C = torch.zeros(plans[0].numel("C"), dtype=torch.float64, device="cuda")
    s = torch.cuda.Stream()
    flops = sum(p.flops for p in plans)
    out = {"extents": ext, "contractions": len(plans), "gflop": flops / 1e9, "c_bytes": C.numel() * 8}
    with torch.cuda.stream(s):
        for _ in range(3):
            tc.execute_group(plans, A, B, C)
        g = torch.cuda.CUDAGraph()
        torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=s):
        tc.execute_group(plans, A, B, C)
    for name, fn in (("eager", lambda: tc.execute_group(plans, A, B, C)), ("graph", g.replay)):
        with torch.cuda.stream(s):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(s)
            for _ in range(reps):
                fn()
            e1.record(s)
            torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / reps
        out[name] = {"ms": round(ms, 4), "tflops": round(flops / ms / 1e9, 2)}
    for beta in (0.0, 1.0):   # one member alone: what beta != 0 (reading C) costs
        with torch.cuda.stream(s):
            plans[0].execute(A[0], B[0], C, 1.0, beta)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(s)
            for _ in range(reps):
                plans[0].execute(A[0], B[0], C, 1.0, beta)
            e1.record(s)
            torch.cuda.synchronize()
        out[f"member0_beta{int(beta)}_ms"] = round(e0.elapsed_time(e1) / reps, 4)
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    torch.cuda.set_device(0)
    run("a:24;b:16;c:16;d:24;e:16;f:16;g:24")
    for n in (16, 24, 32):
        run(";".join(f"{c}:{n}" for c in "abcdefg"))
