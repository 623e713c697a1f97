import sys, numpy as np, torch
sys.path.insert(0, ".")
import oracle, tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from tests.test_gpu_bf16 import _dev_bf16
for var, expr, ext in [(11, "ab-ac-cb", "a:200;b:150;c:130"), (12, "ab-ac-cb", "a:200;b:150;c:130"),
                       (11, "ab-ac-cb", "a:256;b:128;c:128"), (11, "ab-ca-bc", "a:256;b:136;c:192")]:
    p = tc.plan(expr, ext, dtype="bf16", variant=var)
    i = p.info()
    A = tcinputs.bf16_bits(tcinputs.integers_np(p.numel("A"), 1)); B = tcinputs.bf16_bits(tcinputs.integers_np(p.numel("B"), 2))
    dA, dB = _dev_bf16(A), _dev_bf16(B)
    dC = torch.full((p.numel("C"),), float("nan"), dtype=torch.bfloat16, device="cuda")
    p.execute(dA, dB, dC); torch.cuda.synchronize()
    got = dC.cpu().view(torch.int16).numpy().view(np.uint16)
    want = oracle.contract(expr, ext, A, B, dtype="bf16")
    e = tcinputs.parse_extents(ext); na = e["a"]
    bad = np.flatnonzero(got != want)
    print(var, expr, ext, "vec", i["vecX"], i["vecY"], "Mt,Nt,Kt", i["Mt"], i["Nt"], i["Kt"], "bad", bad.size, "of", got.size)
    if bad.size:
        a, b = bad % na, bad // na
        print("  rows", np.unique(a)[:40], "\n  cols", np.unique(b)[:40])
        print("  got", got[bad[:8]], "want", want[bad[:8]])
