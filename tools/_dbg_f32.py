import sys, numpy as np, torch
sys.path.insert(0, ".")
import oracle, tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
torch.cuda.set_device(0)
for dt, var, expr, ext in [("bf16", 11, "ab-ac-cb", "a:200;b:150;c:130"),
                           ("tf32", 21, "ab-ac-cb", "a:128;b:64;c:32"),
                           ("tf32", 21, "ab-ca-cb", "a:128;b:64;c:32"),
                           ("tf32", 21, "ab-ac-bc", "a:128;b:64;c:32"),
                           ("tf32", 21, "ab-ca-bc", "a:128;b:64;c:32"),
                           ("tf32", 22, "ab-ca-bc", "a:128;b:128;c:64"),
                           ("f32", 23, "ab-ca-bc", "a:128;b:64;c:32"),
                           ("f32", 23, "ab-ac-cb", "a:200;b:150;c:130")]:
    try:
        p = tc.plan(expr, ext, dtype=dt, variant=var)
        i = p.info()
        tdt = torch.bfloat16 if dt == "bf16" else torch.float32
        A = tcinputs.integers_np(p.numel("A"), 1); B = tcinputs.integers_np(p.numel("B"), 2)
        dA = torch.tensor(A).to(tdt).cuda(); dB = torch.tensor(B).to(tdt).cuda()
        dC = torch.full((p.numel("C"),), float("nan"), dtype=tdt, device="cuda")
        p.execute(dA, dB, dC); torch.cuda.synchronize()
        got = dC.float().cpu().numpy().astype(np.float64)
        want = oracle.contract(expr, ext, A, B)
        e = tcinputs.parse_extents(ext); na = e["a"]
        bad = np.flatnonzero(got != want)
        print(dt, var, expr, ext, "vec", i["vecX"], i["vecY"], i["vecC"], "kmaj", i["xKmajor"], i["yKmajor"], "bad", bad.size, "of", got.size, flush=True)
        if bad.size:
            a, b = bad % na, bad // na
            print("  rows", np.unique(a)[:40], "\n  cols", np.unique(b)[:40])
            print("  got", got[bad[:8]], "want", want[bad[:8]])
            # is got a permutation-ish of want? check got/want ratios at the first rows
            print("  got[:16]", got[:16], "\n  want[:16]", want[:16], flush=True)
    except Exception as ex:
        print(dt, var, expr, "EXC", ex, flush=True)
        break
