"""Run single BF16 TMA-operand plans in subprocesses (a sticky CUDA error ends only that one)."""
import subprocess
import sys
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys
sys.path.insert(0, "%s")
import numpy as np, torch
import oracle, tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
expr, ext, tiles, var = sys.argv[1:5]
kw = {}
if tiles != "-": kw["force_tiles"] = tiles
if var != "-": kw["variant"] = int(var)
p = tc.plan(expr, ext, dtype="bf16", **kw)
i = p.info()
A = tcinputs.bf16_bits(tcinputs.integers_np(p.numel("A"), 1)); B = tcinputs.bf16_bits(tcinputs.integers_np(p.numel("B"), 2))
dA = torch.from_numpy(A.view(np.int16).copy()).view(torch.bfloat16).cuda()
dB = torch.from_numpy(B.view(np.int16).copy()).view(torch.bfloat16).cuda()
dC = torch.full((p.numel("C"),), float("nan"), dtype=torch.bfloat16, device="cuda")
p.execute(dA, dB, dC); torch.cuda.synchronize()
got = dC.cpu().view(torch.int16).numpy().view(np.uint16)
want = oracle.contract(expr, ext, A, B, dtype="bf16")
print("tma", i["tma_operands"], "tiles", [(x["name"], x["tile"]) for x in i["indices"]], "var", i["variant"], "bad", int((got != want).sum()))
''' % ROOT
cases = [l.split() for l in sys.stdin if l.strip()]
for c in cases:
    r = subprocess.run([sys.executable, "-c", CHILD] + c, capture_output=True, text=True, timeout=120)
    out = (r.stdout.strip().splitlines() or [""])[-1]
    err = [l for l in r.stderr.splitlines() if "Error" in l][-1:] 
    print(" ".join(c), "->", out, err, flush=True)
