"""Sweep of streaming-path tile shapes (kernel_stream.cuh) on TCCG #1-8: a side build with
-DTC_STREAM_DEV reads TC_STREAM_FORCE="<T_a>,<T_E>,<AR>,<KB>,<prod of the other m tiles>" in the
planner; every shape whose tiles divide the extents is timed (L2 flushed, median of 5).
usage: python tools/stream_sweep.py build | run [ids]   (run sets LIBTC_SO itself)"""
import itertools
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
SO = os.path.join(ROOT, "paper_conf_cgo_kimstkpprs19_b200", "build", "sdev", "libtc.so")

if sys.argv[1] == "build":
    from paper_conf_cgo_kimstkpprs19_b200 import build as b
    b.NVCC_FLAGS = list(b.NVCC_FLAGS) + ["-DTC_STREAM_DEV"]
    b.SO = SO
    os.makedirs(os.path.dirname(SO), exist_ok=True)
    b.build(force=True)
    sys.exit(0)

os.environ["LIBTC_SO"] = SO
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


def divs(n, step):
    return [t for t in range(step, min(n, 128) + 1, step) if n % t == 0 or t in (16, 32, 64)]


flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ids = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else list(range(1, 9))
hbm = 6548.8
for c in [c for c in tcinputs.tccg48() if c.id in ids]:
    os.environ.pop("TC_STREAM_FORCE", None)
    p0 = tc.plan(c.expr, c.extents, "bf16", stream=True)
    s0 = p0.info()["stream"]
    ext = dict(kv.split(":") for kv in c.extents.split(";"))
    ext = {k: int(v) for k, v in ext.items()}
    A = tcinputs.uniform(p0.numel("A"), 1000 + c.id, device="cuda").to(torch.bfloat16)
    B = tcinputs.uniform(p0.numel("B"), 2000 + c.id, device="cuda").to(torch.bfloat16)
    C = torch.empty(p0.numel("C"), dtype=torch.bfloat16, device="cuda")
    by = 2 * (p0.numel("A") + p0.numel("B") + p0.numel("C"))
    info = p0.info()
    names = {i["name"]: i for i in info["indices"]}
    Cidx = info["tensors"]["C"]["idx"]
    X = s0["X"]
    Xidx = info["tensors"][X]["idx"]
    a = Cidx[0]
    k = [n for n in Xidx if names[n]["cls"] == "int"][0]
    E = Xidx[0] if Xidx[0] not in (a, k) else None
    rest = [n for n in Xidx if n not in (a, k, E)]
    K = names[k]["n"]
    rps = sorted({r for r in itertools.product(*[divs(names[n]["n"], 1) for n in rest]) if 1})
    rprods = sorted({int(__import__("math").prod(r)) for r in itertools.product(*[[1, 2, 4, 8, 16] for n in rest])})
    res = []
    for ta in divs(names[a]["n"], 8):
        for te in (divs(names[E]["n"], 8) if E else [1]):
            for AR in (4, 8):
                for kb in (16, 32, 64):
                    if kb > -(-K // 16) * 16:
                        continue
                    for rp in rprods:
                        f = f"{ta},{te},{AR},{kb},{rp}"
                        os.environ["TC_STREAM_FORCE"] = f
                        try:
                            p = tc.plan(c.expr, c.extents, "bf16", stream=True)
                        except Exception:  # noqa: BLE001
                            continue
                        s = p.info()["stream"]
                        if not s["on"]:
                            continue
                        ms = timeit(lambda: p.execute(A, B, C), flush)
                        res.append((ms, f, s["units"], s["stages"]))
    res.sort()
    print(json.dumps({"id": c.id, "default": [s0.get("tiles"), s0.get("AR"), s0.get("KB")],
                      "best": [(round(m, 4), f, u, st, round(by / (m * 1e-3) / 1e9 / hbm, 3)) for m, f, u, st in res[:8]],
                      "n": len(res)}), flush=True)
