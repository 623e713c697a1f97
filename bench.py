"""bench.py — TCCG-48 GFLOP/s geomean (FP64) on B200 through libtc's C ABI.

Contract:
  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl libtc|reference] [--cases 1,2,..]
One STEP = one pass of the hot path over the whole workload: all 48 TCCG contractions
(SURVEY.md Appendix A extents, FP64, alpha = 1, beta = 0), inputs resident in HBM, one
tc_execute each.  L2 is flushed (256 MiB memset) before every launch, outside the events.
value = geomean over the 48 cases of 2*prod(N) / (median device time of that case) —
the BASELINE.json metric.  N > 1 (torchrun): every case is C-slab sharded on its largest
external index; A and B are broadcast from rank 0 over NCCL inside the timed
region; time = max over ranks; scaling "strong".
--impl reference: the CPU oracle (oracle/, the paper's plain nested loop) on this box's host
cores, on a bounded sample of the same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import tcinputs  # noqa: E402

METRIC = "TCCG-48 GFLOP/s geomean (FP64) at 1 GPU; % of FP64/tensor peak or HBM roofline"
UNIT = "GFLOP/s"
FP64_PEAK_TFLOPS = 37.16      # measured DMMA peak, profiles/r01_peaks.json (tools/peaks.cu)
# tensor-pipe peaks per dtype: MEASURED_PEAKS.json's dense BF16 (cuBLAS) figure; TF32 runs at
# half the BF16 rate (the guide's nominal ratio), FP32 as split TF32 issues three TF32 MMAs
TENSOR_PEAK_TFLOPS = {"bf16": 1645.0, "tf32": 822.5, "f32": 822.5 / 3}
FP64_PEAK_DERIVED = 148 * 64 * 2 * 1.965e9 / 1e12   # 37.2: SMs x FMA/clk x 2 x max clock


def geomean(xs):
    return math.exp(sum(math.log(x) for x in xs) / len(xs))


def parse_args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="libtc", choices=["libtc", "reference"])
    ap.add_argument("--cases", default="")
    ap.add_argument("--cost", default="b200", choices=["b200", "paper"])
    ap.add_argument("--tune", type=int, default=8,
                    help="measured tuning (tc_plan_tuned) over the model's top-k variants; 0 = model only")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=15.0, help="seconds of oracle work")
    ap.add_argument("--suites", default="ccsdt,membound,triples,eq1graph",
                    help="extra workloads reported inside the same JSON line (BASELINE configs 3/4): "
                         "ccsdt = CCSD(T) 6D sweep N=24..48 FP64, membound = memory-bound TCCG cases in "
                         "FP32 (split TF32) / TF32 / BF16 vs the HBM roofline, triples = the 18 CCSD(T) "
                         "contractions into one t3 (tc_execute_group); '' = none")
    ap.add_argument("--no-splitk", action="store_true", help="skip the split-K demo (SURVEY 8(e))")
    ap.add_argument("--no-scale6d", action="store_true",
                    help="skip the config-5 6D contraction (sd_t_d2, N = 40) timed at every world size")
    ap.add_argument("--profile", action="store_true",
                    help="after the timed region, launch every case once inside cudaProfilerStart/Stop "
                         "(for `ncu --profile-from-start off`); writes gpurun_out/profile_cases.json")
    return ap.parse_args()


def select_cases(spec):
    cases = tcinputs.tccg48()
    if spec:
        ids = {int(x) for x in spec.split(",")}
        cases = [c for c in cases if c.id in ids]
    return cases


# ---------------------------------------------------------------- oracle (CPU) timing
def oracle_sample_rates(cases, budget_s, nthreads=0):
    """Oracle GFLOP/s per case on a contiguous C range sized to ~budget/len(cases) s."""
    import numpy as np
    import oracle
    per = budget_s / len(cases)
    rates = {}
    for c in cases:
        ca, aa, ba = tcinputs.split_expr(c.expr)
        ext = c.ext
        nA, nB, nC = (tcinputs.numel(aa, ext), tcinputs.numel(ba, ext), tcinputs.numel(ca, ext))
        K = 1
        for x in aa:
            if x not in ca:
                K *= ext[x]
        A = tcinputs.uniform_np(nA, 1000 + c.id)
        B = tcinputs.uniform_np(nB, 2000 + c.id)
        n = max(1, min(nC, 2048))
        t0 = time.perf_counter()
        oracle.contract(c.expr, c.extents, A, B, lo=0, hi=n, nthreads=nthreads)
        dt = time.perf_counter() - t0
        n2 = int(min(nC, max(n, n * per / max(dt, 1e-4))))
        t0 = time.perf_counter()
        oracle.contract(c.expr, c.extents, A, B, lo=0, hi=n2, nthreads=nthreads)
        dt = time.perf_counter() - t0
        rates[c.id] = (2.0 * K * n2 / dt / 1e9, n2, nC)
    return rates


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    cases = select_cases(args.cases)
    cores = len(os.sched_getaffinity(0))
    per_step = max(2.0, 150.0 / max(1, args.steps + args.warmup))
    for _ in range(args.warmup):
        oracle_sample_rates(cases, per_step / 4)
    t0 = time.perf_counter()
    vals = []
    for _ in range(args.steps):
        r = oracle_sample_rates(cases, per_step)
        vals.append(geomean([v[0] for v in r.values()]))
    wall = time.perf_counter() - t0
    v = geomean(vals)
    line = {"impl": "reference", "metric": METRIC, "value": round(v, 4), "unit": UNIT,
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(wall / args.steps * 1e3, 1), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "TCCG-48 suite (SURVEY App. A extents), FP64, alpha=1, beta=0",
                       "cases": len(cases)},
            "cpu_baseline": {"value": round(v, 4), "unit": UNIT, "cores": cores, "kind": "oracle",
                             "threads": oracle.max_threads(),
                             "sample": f"per case a contiguous range of C linear indices sized to "
                                       f"~{per_step / len(cases):.2f}s of oracle work per step"},
            "e2e": {"value": round(v, 4), "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- clocks
class Clocks:
    """nvidia-smi sampler (B200_PROFILING.md clocks line).  Started BEFORE the warm-up (the
    tool needs ~1 s to start); each line is stamped on arrival and only the lines that arrive
    inside [mark_start, mark_end] (the timed region) are summarised."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, path):
        self.path = path
        self.p = None
        self.rows = []          # (time, fields)
        self.t0 = self.t1 = None

    def __enter__(self):
        import threading
        try:
            self.p = subprocess.Popen(["nvidia-smi", "--query-gpu=" + self.FIELDS,
                                       "--format=csv,noheader,nounits", "-lms", "50"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None
            return self

        def reader():
            for line in self.p.stdout:
                self.rows.append((time.perf_counter(), line.strip()))
        self.th = threading.Thread(target=reader, daemon=True)
        self.th.start()
        t = time.perf_counter()
        while not self.rows and time.perf_counter() - t < 15 and self.p.poll() is None:
            time.sleep(0.05)
        return self

    def mark_start(self):
        self.t0 = time.perf_counter()

    def mark_end(self):
        self.t1 = time.perf_counter()
        if self.p:
            time.sleep(0.06)

    def __exit__(self, *a):
        if self.p:
            self.p.terminate()
            self.p.wait()
            self.th.join(timeout=2)
        try:
            with open(self.path, "w") as f:
                for t, line in self.rows:
                    inside = self.t0 is not None and self.t0 <= t <= (self.t1 or t)
                    f.write(f"{t:.3f},{int(inside)},{line}\n")
        except Exception:
            pass

    def summary(self, dev=0):
        rows = []
        for t, line in self.rows:
            if self.t0 is None or not (self.t0 <= t <= (self.t1 or t)):
                continue
            r = [x.strip() for x in line.split(",")]
            if len(r) >= 9 and r[0] == str(dev):
                rows.append(r)
        if not rows:
            return None
        sm = sorted(float(r[1]) for r in rows)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower() == "active"})
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": float(rows[0][2]), "reasons": reasons,
                "samples": len(rows), "power_w_max": max(float(r[3]) for r in rows)}


# ---------------------------------------------------------------- GPU run
# ---------------------------------------------------------------- extra suites (configs 3, 4)
_TDT = {"f64": "float64", "f32": "float32", "tf32": "float32", "bf16": "bfloat16"}
_ES = {"f64": 8, "f32": 4, "tf32": 4, "bf16": 2}


def time_one(p, A, B, C, steps, warmup, flush, stream, beta=0.0):
    """Median device time (ms) of one tc_execute over `steps` launches, CUDA events on the
    launch stream, L2 flushed (outside the events) before every launch."""
    import torch
    ts = []
    for i in range(warmup + steps):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        p.execute(A, B, C, beta=beta)
        e1.record(stream)
        e1.synchronize()
        if i >= warmup:
            ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2]


def run_triples(args, flush, stream, dev, hbm):
    """CCSD(T) triples: the 18 sd_t_d1 / sd_t_d2 contractions of TCCG-48
    (#31-48) summed into one t3, FP64, at the TCCG extents and at uniform N.  `fused` = ONE
    kernel (tc_group_plan / tc_group_execute: each t3 tile kept on chip across the 18 members,
    written once), at beta = 0 and beta = 1 (t3 accumulation); `unfused` = the 18
    launches of tc_execute_group (t3 read and written by every member), members tuned top-k at
    their own beta.  The roofline is the fused ideal: min(FP64 peak, I * HBM) with the inputs
    read once and t3 written once (plus read once at beta = 1)."""
    import torch
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    exprs = [c.expr for c in tcinputs.tccg48() if c.group.startswith("CCSDT")]

    def timed(fn, reps):
        ts = []
        for it in range(2 + reps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            e1.synchronize()
            if it >= 2:
                ts.append(e0.elapsed_time(e1))
        return sorted(ts)[len(ts) // 2]

    rows = []
    tccg = [c for c in tcinputs.tccg48() if c.id == 31][0].extents
    for ext in (tccg, ";".join(f"{x}:16" for x in "abcdefg"), ";".join(f"{x}:24" for x in "abcdefg")):
        plans = [tc.plan(e, ext, cost=args.cost) for e in exprs]
        A = [tcinputs.uniform(p.numel("A"), 1000 + i, device=dev) for i, p in enumerate(plans)]
        B = [tcinputs.uniform(p.numel("B"), 2000 + i, device=dev) for i, p in enumerate(plans)]
        C = torch.zeros(plans[0].numel("C"), dtype=torch.float64, device=dev)
        flops = sum(p.flops for p in plans)
        inb = 8 * sum(p.numel("A") + p.numel("B") for p in plans)
        reps = max(3, min(args.steps, 10))
        g = tc.plan_group(plans)
        row = {"extents": ext, "contractions": len(plans), "fused_tile": g.info()["T"],
               "fused_tma": g.info()["tma"], "fused_plan_ms": round(g.info()["plan_ms"], 2)}
        for beta in (0.0, 1.0):
            ms = timed(lambda: g.execute(A, B, C, 1.0, beta), reps)
            attain = min(FP64_PEAK_TFLOPS * 1e12, flops / (inb + 8 * C.numel() * (1 + (beta != 0))) * hbm)
            b = int(beta)
            row[f"fused_ms_b{b}"] = round(ms, 4)
            row[f"fused_gflops_b{b}"] = round(flops / ms / 1e6, 2)
            row[f"fused_roofline_frac_b{b}"] = round(flops / (ms * 1e-3) / attain, 4)
        if args.tune > 0:   # member 0 writes t3 (beta = 0); the rest accumulate: tuned at beta = 1
            plans = [p.tuned(A[i], B[i], C, topk=args.tune, reps=2, beta=0.0 if i == 0 else 1.0)
                     for i, p in enumerate(plans)]
        ms = timed(lambda: tc.execute_group(plans, A, B, C), 3)
        attain = min(FP64_PEAK_TFLOPS * 1e12, flops / (inb + 8 * C.numel()) * hbm)
        row["unfused_ms"] = round(ms, 4)
        row["unfused_gflops"] = round(flops / ms / 1e6, 2)
        row["unfused_roofline_frac_vs_fused"] = round(flops / (ms * 1e-3) / attain, 4)
        row["fused_speedup"] = round(ms / row["fused_ms_b0"], 2)
        rows.append(row)
        del A, B, C, plans, g
        torch.cuda.empty_cache()
    return {"workload": "CCSD(T) triples: TCCG-48 #31-48 into one t3, FP64, at the TCCG extents "
                        "and all extents N; fused = one tc_group_execute kernel (beta 0 / 1), "
                        "unfused = tc_execute_group (18 launches, members tuned at their beta); "
                        "L2 flushed before each group",
            "cases": rows}


def run_eq1_graph(args, stream, dev):
    """BASELINE config 1 / SURVEY 8(d): eq. (1), all extents 16, FP64 — 100 tc_execute launches
    captured in one CUDA graph and replayed (the launch-bound regime), against the same 100
    launches issued eagerly; device time per launch in microseconds, GFLOP/s."""
    import torch
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    p = tc.plan(tcinputs.EQ1_EXPR, tcinputs.EQ1_EXTENTS)
    A = tcinputs.uniform(p.numel("A"), 11, device=dev)
    B = tcinputs.uniform(p.numel("B"), 12, device=dev)
    C = torch.empty(p.numel("C"), dtype=torch.float64, device=dev)
    n = 100
    s2 = torch.cuda.Stream(device=dev)
    s2.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s2):
        for _ in range(3):
            p.execute(A, B, C)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s2):
            for _ in range(n):
                p.execute(A, B, C)
    torch.cuda.current_stream().wait_stream(s2)
    torch.cuda.synchronize()

    def timed(fn, reps):
        ts = []
        for _ in range(reps + 2):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        ts = sorted(ts[2:])
        return ts[len(ts) // 2]

    def eager():
        for _ in range(n):
            p.execute(A, B, C)
    tg = timed(g.replay, max(3, min(args.steps, 10)))
    te = timed(eager, max(3, min(args.steps, 10)))
    return {"workload": "eq.(1) abcd-aebf-dfce, all extents 16, FP64: 100 launches per CUDA graph",
            "us_per_launch_graph": round(1e3 * tg / n, 3), "gflops_graph": round(p.flops * n / tg / 1e6, 2),
            "us_per_launch_eager": round(1e3 * te / n, 3), "gflops_eager": round(p.flops * n / te / 1e6, 2),
            "launches": n, "variant": p.info()["variant"]}


def run_splitk(args, world, rank, sharded, flush, stream, dev, hbm):
    """SURVEY 8(e) split-K demo: ab-ac-cb, a = b = 256, c = 2^20 (the external space fills
    only 4 x 148 SMs' worth of 128 x 128 tiles): at N GPUs each rank contracts its k-range
    and the partials are summed by one NCCL reduce-scatter (|C| / N per rank); FP64, and BF16
    with FP32 partials rounded once (out_f32 + tc_round_bf16).  Inputs are generated
    resident on every rank (this case's exchange step is the reduce-scatter, timed); time =
    max over ranks; HBM roofline on the algorithmic bytes of one GPU's share."""
    import torch
    import torch.distributed as dist
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    from paper_conf_cgo_kimstkpprs19_b200 import dist as tcdist
    expr, extents = "ab-ac-cb", "a:256;b:256;c:1048576"
    n = 256 * 256
    out = {"workload": "split-K ab-ac-cb a=b=256 c=2^20 (NCCL reduce-scatter at N > 1)", "n_gpus": world}
    for dt in ("f64", "bf16"):
        tdt = torch.float64 if dt == "f64" else torch.bfloat16
        base = tc.plan(expr, extents, dtype=dt, out_f32=(dt == "bf16"))
        sub, k, lo, ln = tcdist.split_k_plan(base, expr, extents, world, rank)
        A = tcinputs.uniform(base.numel("A"), 31, device=dev).to(tdt)
        B = tcinputs.uniform(base.numel("B"), 32, device=dev).to(tdt)
        pdt = torch.float64 if dt == "f64" else torch.float32
        Cp = torch.zeros(tcdist.partial_numel(n, world), dtype=pdt, device=dev)
        res = torch.empty(n, dtype=torch.bfloat16, device=dev) if dt == "bf16" else None
        ts = []
        for it in range(args.warmup + max(3, min(args.steps, 5))):
            flush.zero_()
            if sharded:
                dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            if sharded:
                tcdist.execute_split_k(sub, A, B, Cp, world, rank, n=n, out_bf16=res)
            else:
                sub.execute(A, B, Cp[:n])
                if res is not None:
                    tc.round_bf16(res, Cp[:n])
            e1.record(stream)
            torch.cuda.synchronize()
            if it >= args.warmup:
                ts.append(e0.elapsed_time(e1))
        t = torch.tensor([sorted(ts)[len(ts) // 2]], dtype=torch.float64, device=dev)
        if sharded:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = t.item()
        es = 8 if dt == "f64" else 2
        byts = es * (256 * 1048576 * 2) / world + (8 if dt == "f64" else 4) * n
        out[dt] = {"ms": round(ms, 4), "gflops": round(base.flops / ms / 1e6, 2),
                   "hbm_frac_per_gpu": round(byts / (ms * 1e-3) / hbm, 4),
                   "partials": "f64" if dt == "f64" else "f32 (out_f32) + tc_round_bf16"}
        del A, B, Cp
        torch.cuda.empty_cache()
    return out


def run_suite(name, args, flush, stream, dev, hbm):
    """One extra workload: per case plan (+ measured top-k tuning like the main suite), time,
    roofline fraction against min(pipe peak, I * HBM) — pipe = FP64 DMMA for f64; the
    memory-bound cases are reported against HBM bandwidth (algorithmic bytes / time)."""
    import torch
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    rows = []
    if name == "triples":
        return run_triples(args, flush, stream, dev, hbm)
    if name == "eq1graph":
        return run_eq1_graph(args, stream, dev)
    if name == "ccsdt":
        # BASELINE config 3: sd_t_d1 / sd_t_d2 6D contractions at uniform extents 24..48, FP64,
        # beta = 0 (t3 written) and beta = 1 (t3 accumulated)
        todo = [(tcinputs.ccsdt(n, e, 100 + n), "f64", beta) for e in ("abcdef-gdab-efgc", "abcdef-dega-gfbc")
                for n in (24, 32, 40, 48) for beta in (0.0, 1.0)]
    else:
        # BASELINE config 4: the memory-bound TCCG cases (#1-8 ML tensor x matrix, #18 ab-ac-cb)
        mb = [c for c in tcinputs.tccg48() if c.id <= 8 or c.id == 18]
        todo = [(c, dt, 0.0) for dt in ("f32", "tf32", "bf16") for c in mb]
    for c, dt, beta in todo:
        tdt = getattr(torch, _TDT[dt])
        p = tc.plan(c.expr, c.extents, dtype=dt, cost=args.cost)
        A = tcinputs.uniform(p.numel("A"), 1000 + c.id, device=dev).to(tdt)
        B = tcinputs.uniform(p.numel("B"), 2000 + c.id, device=dev).to(tdt)
        C = torch.zeros(p.numel("C"), dtype=tdt, device=dev) if beta else torch.empty(p.numel("C"), dtype=tdt, device=dev)
        if args.tune > 0:
            p = p.tuned(A, B, C, topk=args.tune, reps=5, beta=beta)
        ms = time_one(p, A, B, C, max(3, min(args.steps, 5)), 2, flush, stream, beta=beta)
        byts = _ES[dt] * (p.numel("A") + p.numel("B") + p.numel("C") * (2 if beta else 1))
        gbs = byts / (ms * 1e-3) / 1e9
        r = {"expr": c.expr, "extents": c.extents, "dtype": dt, "beta": beta, "ms": round(ms, 5),
             "gflops": round(p.flops / ms / 1e6, 2), "gbs": round(gbs, 1),
             "variant": "stream" if p.info()["stream"].get("active", 0) == 1 else p.info()["variant"]}
        if dt == "f64":
            attain = min(FP64_PEAK_TFLOPS * 1e12, p.flops / byts * hbm)
            r["roofline_frac"] = round(p.flops / (ms * 1e-3) / attain, 4)
        else:
            r["hbm_frac"] = round(gbs * 1e9 / hbm, 4)
            # tensor-pipe peak of the dtype (MEASURED_PEAKS.json BF16 cuBLAS figure; TF32 half of
            # it; FP32 = three TF32 MMAs per product): #18 is compute-bound, judged against it
            pk = TENSOR_PEAK_TFLOPS[dt] * 1e12
            r["roofline_frac"] = round(p.flops / (ms * 1e-3) / min(pk, p.flops / byts * hbm), 4)
            r["bound"] = "tensor" if p.flops / byts * hbm > pk else "hbm"
            r["cta_pair"] = p.info().get("cta_pair", 0)
            r["tma_operands"] = p.info().get("tma_operands", 0)
        rows.append(r)
        del A, B, C, p
        torch.cuda.empty_cache()
    out = {"cases": rows}
    if name == "ccsdt":
        out["workload"] = "CCSD(T) sd_t_d2 abcdef-gdab-efgc and sd_t_d1 abcdef-dega-gfbc, all extents N, FP64"
        for b in (0.0, 1.0):
            sel = [r for r in rows if r["beta"] == b]
            out[f"geomean_gflops_beta{int(b)}"] = round(geomean([r["gflops"] for r in sel]), 2)
            out[f"geomean_roofline_frac_beta{int(b)}"] = round(geomean([r["roofline_frac"] for r in sel]), 4)
    else:
        out["workload"] = ("memory-bound TCCG #1-8 in FP32 (split TF32), TF32, BF16 against HBM; #18 "
                           "ab-ac-cb (compute-bound) reported apart against the dtype's tensor peak")
        for dt in ("f32", "tf32", "bf16"):
            sel = [r for r in rows if r["dtype"] == dt and r["expr"] != "ab-ac-cb"]
            out[f"geomean_hbm_frac_{dt}"] = round(geomean([r["hbm_frac"] for r in sel]), 4)
            out[f"geomean_gflops_{dt}"] = round(geomean([r["gflops"] for r in sel]), 2)
            g = [r for r in rows if r["dtype"] == dt and r["expr"] == "ab-ac-cb"]
            if g:
                out[f"ab_ac_cb_{dt}"] = {"tflops": round(g[0]["gflops"] / 1e3, 1),
                                         "tensor_peak_frac": g[0]["roofline_frac"],
                                         "peak_tflops": TENSOR_PEAK_TFLOPS[dt]}
    return out


def run_libtc(args):
    import torch
    import torch.distributed as dist
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    from paper_conf_cgo_kimstkpprs19_b200 import dist as tcdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    # the sharded path (C slabs + NCCL input broadcast); TC_BENCH_FORCE_DIST=1 takes it at
    # world size 1 too (a one-GPU check of the multi-GPU code path under torchrun)
    sharded = world > 1 or os.environ.get("TC_BENCH_FORCE_DIST") == "1"
    torch.cuda.set_device(local)
    if sharded:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    cases = select_cases(args.cases)
    dev = torch.device("cuda", local)

    def kname(p):
        i = p.info()
        s = i["stream"]
        if s.get("active"):   # the streaming path (stream.hpp)
            return f"tc_stream_f64_kernel<{s['NB']},{s['AR']},{'true' if s['mode'] == 'T' else 'false'}>"
        return (f"tc_f64_dmma_kernel<{i['BM']},{i['BN']},{i['BK']},{i['WM']},{i['WN']},{i['stages']},4,"
                f"{i['occ']},{i['xKmajor']},{i['yKmajor']},{i['stg']}>")

    stream = torch.cuda.current_stream()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    # plans + resident inputs (rank 0's inputs are the source of the broadcast at N > 1)
    work = []
    model_pick = {}   # case id -> the cost model's own (untuned) plan
    t_plan = t_tune = 0.0
    for c in cases:
        t0 = time.perf_counter()
        p = tc.plan(c.expr, c.extents, cost=args.cost)
        if sharded:
            sh = tcdist.shard_plan(p, c.expr, c.extents, world, rank)
        t_plan += time.perf_counter() - t0
        A = tcinputs.uniform(p.numel("A"), 1000 + c.id, device=dev)
        B = tcinputs.uniform(p.numel("B"), 2000 + c.id, device=dev)
        model_pick[c.id] = p
        if not sharded:
            C = torch.empty(p.numel("C"), dtype=torch.float64, device=dev)
            if args.tune > 0:
                t0 = time.perf_counter()
                p = p.tuned(A, B, C, topk=args.tune, reps=5)
                t_tune += time.perf_counter() - t0
            work.append((c, p, A, B, C, None))
        else:
            if sh.x_tensor is not None and rank != 0:   # the scattered input: this rank's slab only
                if sh.x_tensor == "A":
                    A = torch.empty(tcdist.local_input_numel(sh, "A", p.numel("A"), rank), dtype=torch.float64, device=dev)
                else:
                    B = torch.empty(tcdist.local_input_numel(sh, "B", p.numel("B"), rank), dtype=torch.float64, device=dev)
            C = torch.empty(sh.c_numel, dtype=torch.float64, device=dev)
            if args.tune > 0 and sh.plan is not None:
                t0 = time.perf_counter()
                sh.plan = sh.plan.tuned(A, B, C, topk=args.tune, reps=5)
                t_tune += time.perf_counter() - t0
            work.append((c, p, A, B, C, sh))

    def one(i, record):
        c, p, A, B, C, sh = work[i]
        flush.zero_()
        if sharded:
            dist.barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        if sh is None:
            p.execute(A, B, C)
        else:
            tcdist.distribute_inputs(sh, A, B, rank, src=0)
            if sh.plan is not None:
                a, b = tcdist.local_operands(sh, A, B, rank)
                sh.plan.execute(a, b, C)
        e1.record(stream)
        record.append((e0, e1))

    clk_path = os.path.join(ROOT, "gpurun_out", f"bench_clocks_r{rank}.csv")
    os.makedirs(os.path.dirname(clk_path), exist_ok=True)
    times = [[] for _ in work]
    with Clocks(clk_path) as clocks:
        for _ in range(args.warmup):
            rec = []
            for i in range(len(work)):
                one(i, rec)
        torch.cuda.synchronize()
        if sharded:
            dist.barrier()
        torch.cuda.synchronize()
        clocks.mark_start()
        t_wall = time.perf_counter()
        for _ in range(args.steps):
            rec = []
            for i in range(len(work)):
                one(i, rec)
            torch.cuda.synchronize()
            for i, (e0, e1) in enumerate(rec):
                times[i].append(e0.elapsed_time(e1))
        if sharded:
            dist.barrier()
        torch.cuda.synchronize()
        t_wall = time.perf_counter() - t_wall
        clocks.mark_end()
    if args.profile and rank == 0:
        # one launch per case inside a profiler range (ncu --profile-from-start off); the
        # order of the captured launches is the order of profile_cases.json
        rows = []
        for (c, p, A, B, C, sh) in work:
            flush.zero_()
            torch.cuda.synchronize()
            torch.cuda.cudart().cudaProfilerStart()
            (sh.plan if sh is not None else p).execute(A, B, C)
            torch.cuda.synchronize()
            torch.cuda.cudart().cudaProfilerStop()
            rows.append({"case": c.id, "kernel": kname((sh.plan if sh is not None else p)),
                         "flops": p.flops,
                         "alg_bytes": 8 * (p.numel("A") + p.numel("B") + p.numel("C"))})
        with open(os.path.join(ROOT, "gpurun_out", "profile_cases.json"), "w") as f:
            json.dump(rows, f)
    med = []
    for ts in times:
        s = sorted(ts)
        med.append(s[len(s) // 2])
    if sharded:
        t = torch.tensor(med, dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        med = t.tolist()
    def run_plan(w):   # the plan that executes (a rank's shard at N > 1)
        return w[5].plan if w[5] is not None and w[5].plan is not None else w[1]

    per_case = []
    for w, ms in zip(work, med):
        c, p = w[0], w[1]
        ri = run_plan(w).info()
        act = ri["stream"].get("active", 0) == 1
        per_case.append({"id": c.id, "ms": round(ms, 5), "gflops": round(p.flops / ms / 1e6, 2),
                         "variant": "stream" if act else ri["variant"],
                         "pred_ms": round(ri["stream"]["t_pred_ms"] if act else ri["t_pred_ms"], 5)})
    value = geomean([r["gflops"] for r in per_case])

    # cost-model fidelity (outside the timed region): the model's predicted time of the plan
    # that ran vs its measured time, and the model's own pick (untuned) timed vs the tuned one
    model = None
    if not sharded:
        errs, picks = [], []
        for w, r in zip(work, per_case):
            r["model_err"] = round(r["pred_ms"] / r["ms"] - 1.0, 4)
            errs.append(abs(r["model_err"]))
            pm = model_pick[w[0].id]
            pmi = pm.info()
            pm_var = "stream" if pmi["stream"].get("active", 0) == 1 else pmi["variant"]
            pm_ms = r["ms"] if pm_var == r["variant"] and run_plan(w) is pm \
                else time_one(pm, w[2], w[3], w[4], 3, 1, flush, stream)
            r["model_pick_ms"] = round(pm_ms, 5)
            picks.append(pm_ms / r["ms"])
        errs.sort()
        model = {"median_abs_err": round(errs[len(errs) // 2], 4),
                 "within_25pct": sum(e <= 0.25 for e in errs), "cases": len(errs),
                 "pick_within_10pct_of_tuned": sum(x <= 1.10 for x in picks),
                 "pick_vs_tuned_geomean": round(geomean(picks), 4),
                 "how": "pred_ms = the B200 cost model's t_pred of the timed plan; model_err = "
                        "pred / measured - 1; model_pick_ms = the untuned plan (the model's "
                        "first choice) timed like the suite (3 launches, L2 flushed)"}
    ms_step = sum(med)

    # dominant kernel (largest share of the step) -> roofline

    share = {}
    for w, ms in zip(work, med):
        c, p = w[0], w[1]
        k = kname(run_plan(w))
        f, t = share.get(k, (0.0, 0.0))
        share[k] = (f + p.flops, t + ms)
    dom = max(share, key=lambda k: share[k][1])
    dflops, dms = share[dom]
    achieved = dflops / (dms * 1e-3) / 1e12
    dom_cases = [w[0].id for w in work if kname(run_plan(w)) == dom]
    # DRAM bytes per launch of the dominant kernel from the committed `ncu --set full` capture
    # (tools/ncu_traffic.py -> profiles/ncu_traffic.json): mean over the dominant cases whose
    # captured kernel is the one that ran here (tuning can pick another variant on another box)
    traffic, traffic_alg = None, None
    prof = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(prof):
        try:
            t = {r["case"]: r for r in json.load(open(prof))["launches"]}
            hit = [t[i] for i in dom_cases if i in t and t[i]["kernel"] == dom]
            if hit:
                traffic = round(sum(r["dram_bytes"] for r in hit) / len(hit))
                traffic_alg = round(sum(r["alg_bytes"] for r in hit) / len(hit))
        except Exception:
            traffic = None
    roof = {"bound": "tensor", "achieved": round(achieved, 3), "peak": FP64_PEAK_TFLOPS,
            "unit": "TFLOP/s", "frac": round(achieved / FP64_PEAK_TFLOPS, 4), "traffic": traffic,
            "kernel": dom, "cases": dom_cases,
            "peak_source": "measured FP64 DMMA peak (tools/peaks.cu, profiles/r01_peaks.json); "
                           f"derived 148x64x2x1.965GHz = {FP64_PEAK_DERIVED:.2f}",
            "traffic_cases": "mean dram__bytes_read+write per launch over the dominant cases "
                             "captured in profiles/ncu_traffic.json",
            "alg_bytes_per_launch": traffic_alg,
            "launches_per_step": len(dom_cases),
            "share_of_step": round(dms / ms_step, 4)}

    # per-class roofline fraction: min(FP64 peak, I * HBM) per case
    hbm = 6554.2e9
    try:
        hbm = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] * 1e9
    except Exception:
        pass
    fr = []
    for (c, p, A, B, C, sh), ms in zip(work, med):
        byts = 8.0 * (p.numel("A") + p.numel("B") + p.numel("C"))
        attain = min(FP64_PEAK_TFLOPS * 1e12, p.flops / byts * hbm)
        fr.append(p.flops / (ms * 1e-3) / attain)
    clk = clocks.summary(local)

    # end-to-end through tc_execute_host (pinned host buffers; copies inside the timing)
    e2e = None
    if not args.no_e2e and world == 1:
        e2e_vals, h2d, d2h = [], 0, 0
        maxA = max(w[1].numel("A") for w in work)
        maxB = max(w[1].numel("B") for w in work)
        maxC = max(w[1].numel("C") for w in work)
        hA = torch.empty(maxA, dtype=torch.float64).pin_memory()
        hB = torch.empty(maxB, dtype=torch.float64).pin_memory()
        hC = torch.empty(maxC, dtype=torch.float64).pin_memory()
        ws = torch.empty(max(w[1].workspace_bytes() for w in work) // 8 + 1, dtype=torch.float64,
                         device=dev)
        for (c, p, A, B, C, sh) in work:
            hA[:A.numel()].copy_(A)
            hB[:B.numel()].copy_(B)
            ts = []
            for r in range(2):
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                p.execute_host(hA, hB, hC, ws)
                ts.append(time.perf_counter() - t0)
            e2e_vals.append(p.flops / min(ts) / 1e9)
            h2d += 8 * (A.numel() + B.numel())
            d2h += 8 * p.numel("C")
        e2e = {"value": round(geomean(e2e_vals), 3), "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h,
               "how": "tc_execute_host per case: pinned host A,B -> device, kernel, C -> host, "
                      "stream sync; wall clock, best of 2"}

    # BASELINE config 5 / SURVEY 8(e): the large 6D contraction (sd_t_d2, all extents 40) sharded
    # on its largest external index — the case the >= 85 % scaling target is stated for.
    # Reported at every N (max over ranks) with and without the input broadcast.
    scale6d = None
    if not args.no_scale6d:
        c6 = tcinputs.ccsdt(40, "abcdef-gdab-efgc", 140)
        p6 = tc.plan(c6.expr, c6.extents, cost=args.cost)
        A6 = tcinputs.uniform(p6.numel("A"), 1140, device=dev)
        B6 = tcinputs.uniform(p6.numel("B"), 2140, device=dev)
        sh6 = tcdist.shard_plan(p6, c6.expr, c6.extents, world, rank) if sharded else None
        run6 = sh6.plan if sh6 is not None else p6
        C6 = torch.empty(sh6.c_numel if sh6 is not None else p6.numel("C"), dtype=torch.float64, device=dev)
        if sh6 is not None and sh6.x_tensor is not None and rank != 0:
            # the scattered input: this rank holds only its slab
            if sh6.x_tensor == "A":
                A6 = torch.empty(tcdist.local_input_numel(sh6, "A", p6.numel("A"), rank), dtype=torch.float64, device=dev)
            else:
                B6 = torch.empty(tcdist.local_input_numel(sh6, "B", p6.numel("B"), rank), dtype=torch.float64, device=dev)
        if args.tune > 0 and run6 is not None:   # the same measured top-k as every other case
            run6 = run6.tuned(A6, B6, C6, topk=args.tune, reps=2)
        tot, comp = [], []
        for it in range(args.warmup + max(3, min(args.steps, 5))):
            flush.zero_()
            if sharded:
                dist.barrier()
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
            ev[0].record(stream)
            if sharded:
                tcdist.distribute_inputs(sh6, A6, B6, rank, src=0)
            ev[1].record(stream)
            if run6 is not None:
                a6, b6 = tcdist.local_operands(sh6, A6, B6, rank) if sh6 is not None else (A6, B6)
                run6.execute(a6, b6, C6)
            ev[2].record(stream)
            torch.cuda.synchronize()
            if it >= args.warmup:
                tot.append(ev[0].elapsed_time(ev[2]))
                comp.append(ev[1].elapsed_time(ev[2]))
        t6 = torch.tensor([sorted(tot)[len(tot) // 2], sorted(comp)[len(comp) // 2]], dtype=torch.float64, device=dev)
        if sharded:
            dist.all_reduce(t6, op=dist.ReduceOp.MAX)
        scale6d = {"expr": c6.expr, "extents": c6.extents, "n_gpus": world,
                   "ms": round(t6[0].item(), 4), "gflops": round(p6.flops / t6[0].item() / 1e6, 2),
                   "ms_compute_only": round(t6[1].item(), 4),
                   "gflops_compute_only": round(p6.flops / t6[1].item() / 1e6, 2),
                   "inputs": ("scatter " + sh6.x_tensor + ", broadcast the other") if sh6 is not None and sh6.x_tensor
                             else "broadcast A and B",
                   "how": "C slab on the largest external index per rank; the input holding it scattered "
                          "as slabs when it is that input's slowest index, else broadcast (NCCL), inside "
                          "the first interval; time = max over ranks (SURVEY 8(e))"}
        del A6, B6, C6
        torch.cuda.empty_cache()

    splitk = None if args.no_splitk else run_splitk(args, world, rank, sharded, flush, stream, dev, hbm)

    suites = {}
    if world == 1 and args.suites:
        for name in args.suites.split(","):
            suites[name] = run_suite(name, args, flush, stream, dev, hbm)

    cpu = None
    if not args.no_cpu and rank == 0 and world == 1:
        import oracle
        rates = oracle_sample_rates(cases, args.cpu_budget)
        cpu = {"value": round(geomean([v[0] for v in rates.values()]), 4), "unit": UNIT,
               "cores": len(os.sched_getaffinity(0)), "threads": oracle.max_threads(),
               "kind": "oracle",
               "sample": f"per case a contiguous range of C linear indices sized to "
                         f"~{args.cpu_budget / len(cases):.2f}s of oracle work "
                         f"({sum(v[1] for v in rates.values())} of "
                         f"{sum(v[2] for v in rates.values())} C elements)",
               "cpu_model": oracle.cpu_model(),
               "build": "gcc -O3 -march=native -fopenmp -ffp-contract=off (oracle/__init__.py)"}
        # single-thread oracle figures on eq. (1) and TCCG #3
        eq1 = tcinputs.Case(0, tcinputs.EQ1_EXPR, tcinputs.EQ1_EXTENTS, "H", "eq1")
        c3 = [c for c in tcinputs.tccg48() if c.id == 3]
        r1 = oracle_sample_rates([eq1] + c3, 4.0, nthreads=1)
        cpu["one_thread_gflops"] = {"eq1_N16": round(r1[0][0], 4), "tccg3": round(r1[3][0], 4)}

    if rank == 0:
        line = {"metric": METRIC, "value": round(value, 2), "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 4),
                "higher_is_better": True, "scaling": "strong" if sharded else "weak",
                "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": "TCCG-48 suite (SURVEY App. A extents), FP64, alpha=1, beta=0",
                           "cases": len(cases), "cost_model": args.cost,
                           "l2": "flushed before every launch (256 MiB memset, outside events)",
                           "timing": "CUDA events per launch on the launch stream; median of steps",
                           "parallelism": f"C-slab shard x{world}" if sharded else "single GPU"},
                "roofline": roof,
                "roofline_geomean_frac": round(geomean(fr), 4),
                # per TCCG class (SURVEY App. A groups): geomean of achieved / min(FP64 peak, I * HBM)
                "roofline_frac_by_class": {
                    name: round(geomean([f for (w, f) in zip(work, fr) if lo <= w[0].id <= hi]), 4)
                    for name, lo, hi in (("memory_bound_1_8", 1, 8), ("compute_bound_9_30", 9, 30),
                                         ("near_ridge_ccsdt_31_48", 31, 48))
                    if any(lo <= w[0].id <= hi for w in work)},
                "cpu_baseline": cpu, "e2e": e2e,
                "gpu_launches": len(work) * args.steps,
                "clocks": clk,
                "plan_ms_total": round(t_plan * 1e3, 2),
                "tune": {"topk": args.tune, "ms_total": round(t_tune * 1e3, 2),
                         "how": "tc_plan_tuned: best config of each of the model's top-k variants and the "
                                "streaming path's three best configs, each launched 1+5 times on the "
                                "case's own tensors after an L2 flush, lowest median kept (outside "
                                "the timed region; P:L346-348)"},
                "wall_s_timed": round(t_wall, 3),
                "suites": suites,
                "scale6d": scale6d,
                "splitk": splitk,
                "cost_model": model,
                "per_case": per_case}
        print(json.dumps(line), flush=True)
    if sharded:
        dist.destroy_process_group()


def main():
    args = parse_args()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_libtc(args)


if __name__ == "__main__":
    main()
