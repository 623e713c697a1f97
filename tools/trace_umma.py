"""Per-stage hand-off timeline of the tcgen05 kernel (-DTC_TRACE side build, CTA 0, clock64).
Builds a -DTC_TRACE libtc on the side (build/trace/libtc.so) and loads it instead.
usage: python tools/trace_umma.py <case> <dtype>"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
# (the side library must be chosen before the package — and its binding — is imported)
_so = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_cgo_kimstkpprs19_b200",
                   "build", "trace", "libtc.so")
os.environ["LIBTC_SO"] = _so
from paper_conf_cgo_kimstkpprs19_b200 import build as _b  # noqa: E402
if not os.path.exists(_so):
    _b.NVCC_FLAGS = _b.NVCC_FLAGS + ["-DTC_TRACE"]
    _b.SO = _so
    os.makedirs(os.path.dirname(_so), exist_ok=True)
    _b.build(force=True)
os.environ["LIBTC_SO"] = _so
import numpy as np  # noqa: E402
import torch  # noqa: E402
import tcinputs  # noqa: E402
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc  # noqa: E402

cid, dt = int(sys.argv[1]), sys.argv[2]
case = [c for c in tcinputs.tccg48() if c.id == cid][0]
tdt = {"bf16": torch.bfloat16, "f32": torch.float32, "tf32": torch.float32}[dt]
p = tc.plan(case.expr, case.extents, dtype=dt)
A = tcinputs.uniform(p.numel("A"), 1, device="cuda").to(tdt)
B = tcinputs.uniform(p.numel("B"), 2, device="cuda").to(tdt)
C = torch.zeros(max(p.numel("C"), 8 * 1024 * 8 // tdt.itemsize + 64), dtype=tdt, device="cuda")
for _ in range(3):
    C.zero_()
    p.execute(A, B, C)
torch.cuda.synchronize()
t = C.view(torch.int64)[:8 * 1024].cpu().numpy().reshape(8, 1024).astype(np.int64)
i = p.info()
ns = i["nsteps"]
t0 = t[0][0]
n = int(np.count_nonzero(t[2]))
print(cid, dt, "variant", i["variant"], "nsteps/tile", ns, "stages traced", n)
names = ["prod_empty_ok", "prod_arrived", "mma_full_ok", "mma_committed", "epi_tfull_ok", "epi_released"]
for j in list(range(0, 12)) + [n // 2, n - 1]:
    row = []
    for k in range(4):
        row.append(f"{names[k]}={t[k][j] - t0:8d}")
    print(f"stage {j:4d} " + " ".join(row))
d = np.diff(t[2][:n])
print("MMA full-to-full per stage: median", int(np.median(d)), "clk; producer arrive-to-arrive:",
      int(np.median(np.diff(t[1][:n]))), "; producer empty-wait ->arrive:", int(np.median((t[1] - t[0])[:n])),
      "; arrive->mma full ok:", int(np.median((t[2] - t[1])[:n])), "; mma ok->committed:", int(np.median((t[3] - t[2])[:n])))
print("arrive -> after tile switch:", int(np.median((t[7] - t[1])[:n - 1])), "; tile switch -> loop top:",
      int(np.median((t[6][1:n] - t[7][:n - 1]))), "; loop top -> empty ok:", int(np.median((t[0] - t[6])[:n])))
nt = int(np.count_nonzero(t[4]))
if nt > 2:
    print("epilogue tiles", nt, "tfull-to-tfull median", int(np.median(np.diff(t[4][:nt]))),
          "; tfull->released", int(np.median((t[5] - t[4])[:nt])))
