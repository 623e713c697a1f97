"""Full-size parity: every workload bench.py times, at its full extents and in the exact
launch configuration bench.py times it in (same planning, same measured top-k tuning, same
seeded device inputs, same alpha / beta), checked against the CPU oracle on sampled outputs:
2^16 random elements plus EVERY element of the first and the last C tile of the plan
(SURVEY 8(d) "Parity for the large cases"), and against the rank-1 closed form on every
output element for a subset.  Needs a B200.

Covered: TCCG-48 FP64 (model plan and tuned plan), the CCSD(T) sweep of config 3 at
N = 24..48 (beta = 0) and TCCG #31-48 at beta = 1 (NWChem-style t3 accumulation),
the memory-bound suite of config 4 (#1-8, #18 in FP32 / TF32 / BF16), the streaming path at
beta != 0 (#1, #3, #7, #10 in FP64 / FP32 / TF32) and the FP32 SD2
family of Figs. 6/7 (sd_t_d2, TCCG #40-48, single precision)."""
import numpy as np
import pytest
import torch

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build

pytestmark = pytest.mark.gpu
TAU64 = 1e-12
NSAMPLE = 1 << 16
TUNE_TOPK = 8          # bench.py --tune default
_TDT = {"f64": torch.float64, "f32": torch.float32, "tf32": torch.float32, "bf16": torch.bfloat16}


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


def tile_indices(p, last: bool) -> np.ndarray:
    """C linear indices of every element of the plan's first (origin) or last C tile, from
    the plan's own (normalised) C view: index extents, tiles and strides (tc_plan_info)."""
    info = p.info()
    ix = {d["name"]: d for d in info["indices"]}
    cv = info["tensors"]["C"]
    off = np.array([cv["base"]], dtype=np.int64)
    for name, stride in zip(cv["idx"], cv["stride"]):
        n, t = ix[name]["n"], max(1, ix[name]["tile"])
        o = (n - 1) // t * t if last else 0
        r = np.arange(o, min(o + t, n), dtype=np.int64) * stride
        off = (off[:, None] + r[None, :]).reshape(-1)
    return off


def sample_indices(p, n: int, seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return np.unique(np.concatenate([rng.integers(0, n, NSAMPLE), tile_indices(p, False),
                                     tile_indices(p, True), np.array([0, n - 1])]))


def check_sampled(p, case, dtype, A, B, C, C0=None, beta=0.0, seed=0):
    """Sampled parity of C (device) against the oracle on the same inputs (upcast exactly)."""
    n = C.numel()
    idx = sample_indices(p, n, seed)
    got = C[torch.as_tensor(idx, device=C.device)].double().cpu().numpy()
    c0 = None if C0 is None else C0.double().cpu().numpy()
    exact, S = oracle.sample(case.expr, case.extents, A.double().cpu().numpy(), B.double().cpu().numpy(),
                             idx, C=c0, beta=beta, with_scale=True)
    K = p.flops / 2 / max(1, p.numel("C"))
    if dtype == "f64":
        tol = TAU64 * S
    elif dtype == "f32":
        tol = 1e-5 * S                                     # north_star FP32
    elif dtype == "tf32":                                  # DESIGN R30
        tol = 2.0 ** -9 * S + 2.0 ** -23 * np.abs(exact)
    else:                                                  # one BF16 ulp + FP32 accumulation
        tol = 2.0 ** -8 * np.abs(exact) + K * 2.0 ** -23 * S
    bad = np.flatnonzero(~(np.abs(got - exact) <= tol))
    assert bad.size == 0, (case.expr, dtype, idx[bad[:5]], got[bad[:5]], exact[bad[:5]], p.info()["variant"])
    return idx.size


def inputs(p, case, dtype, dev="cuda"):
    tdt = _TDT[dtype]
    A = tcinputs.uniform(p.numel("A"), 1000 + case.id, device=dev).to(tdt)
    B = tcinputs.uniform(p.numel("B"), 2000 + case.id, device=dev).to(tdt)
    return A, B


def run_tuned(case, dtype="f64", beta=0.0, tune=True):
    """Plan + tune exactly as bench.py does, then one execute on NaN-prefilled C (beta = 0) or
    on the seeded C_in (beta != 0); returns what check_sampled needs."""
    tdt = _TDT[dtype]
    p = tc.plan(case.expr, case.extents, dtype=dtype)
    A, B = inputs(p, case, dtype)
    C = torch.empty(p.numel("C"), dtype=tdt, device="cuda")
    C0 = None
    if beta != 0.0:
        C0 = tcinputs.uniform(p.numel("C"), 3000 + case.id, device="cuda").to(tdt)
    if tune:
        if beta != 0.0:
            C.copy_(C0)
        p = p.tuned(A, B, C, topk=TUNE_TOPK, reps=1, beta=beta)
    if beta != 0.0:
        C.copy_(C0)
    else:
        C.fill_(float("nan"))
    p.execute(A, B, C, beta=beta)
    torch.cuda.synchronize()
    return p, A, B, C, C0


@pytest.mark.parametrize("tuned", [False, True], ids=["model", "tuned"])
@pytest.mark.parametrize("case", tcinputs.tccg48(), ids=lambda c: f"tccg{c.id}")
def test_tccg_full_size_sampled(case, tuned):
    p, A, B, C, _ = run_tuned(case, tune=tuned)
    check_sampled(p, case, "f64", A, B, C, seed=case.id)
    assert torch.isfinite(C).all()          # every element was written
    del A, B, C


@pytest.mark.parametrize("case", [c for c in tcinputs.tccg48() if c.id >= 31], ids=lambda c: f"tccg{c.id}")
def test_ccsdt_tccg_beta1_tuned(case):
    # CCSD(T) sd_t_d1 / d2 accumulating into t3 (beta = 1),
    # planned and tuned at beta = 1 as bench.py's ccsdt suite and the triples group run them
    p, A, B, C, C0 = run_tuned(case, beta=1.0)
    check_sampled(p, case, "f64", A, B, C, C0=C0, beta=1.0, seed=case.id)


@pytest.mark.parametrize("dtype", ["f64", "f32", "tf32"])
@pytest.mark.parametrize("cid", [1, 3, 7, 10])
def test_stream_full_size_beta(dtype, cid):
    # the streaming path's beta != 0 instances (kernels_stream_beta.cu: old C read once per
    # element in the store phase) at full TCCG extents: SM_T (#1, #3), SM_K (#7), SM_M (#10,
    # FP64 only), C = alpha * A.B + beta * C_in
    case = [c for c in tcinputs.tccg48() if c.id == cid][0]
    p = tc.plan(case.expr, case.extents, dtype=dtype, stream=True)
    if p.info()["stream"]["on"] != 1:
        pytest.skip(f"not a streaming shape in {dtype}: {p.info()['stream']['why']}")
    assert p.info()["stream"]["active"] == 1
    A, B = inputs(p, case, dtype)
    C0 = tcinputs.uniform(p.numel("C"), 3000 + case.id, device="cuda").to(_TDT[dtype])
    C = C0.clone()
    p.execute(A, B, C, beta=-0.5)
    torch.cuda.synchronize()
    check_sampled(p, case, dtype, A, B, C, C0=C0, beta=-0.5, seed=100 + cid)


# (beta = 1 rows at N <= 32: the oracle needs the whole C_in on the host, and at N = 48 a
# second 97.8 GB C_in does not fit the GPU next to C)
@pytest.mark.parametrize("n,beta", [(24, 0.0), (32, 0.0), (40, 0.0), (48, 0.0), (24, 1.0), (32, 1.0)])
@pytest.mark.parametrize("expr", ["abcdef-gdab-efgc", "abcdef-dega-gfbc"])
def test_ccsdt_sweep_tuned(expr, n, beta):
    # bench.py's ccsdt suite (BASELINE config 3), each row in its own launch configuration
    case = tcinputs.ccsdt(n, expr, 100 + n)
    p, A, B, C, C0 = run_tuned(case, beta=beta)
    check_sampled(p, case, "f64", A, B, C, C0=C0, beta=beta, seed=n)
    if beta == 0.0:
        assert not bool(torch.isnan(C).any())
    del A, B, C, C0
    torch.cuda.empty_cache()


@pytest.mark.parametrize("n,expr", [(48, "abcdef-gdab-efgc"), (40, "abcdef-dega-gfbc")])
def test_ccsdt_max_size_int64_offsets(n, expr):
    # |C| = 48^6 = 1.2e10 FP64 elements (97.8 GB), past 2^31: every 64-bit offset path of the
    # tables and the epilogue runs; elements around 2^31 and 2^32 are sampled explicitly
    case = tcinputs.ccsdt(n, expr, 100 + n)
    p = tc.plan(case.expr, case.extents)
    A, B = inputs(p, case, "f64")
    C = torch.full((p.numel("C"),), float("nan"), dtype=torch.float64, device="cuda")
    p.execute(A, B, C)
    torch.cuda.synchronize()
    nC = C.numel()
    extra = [(np.int64(1) << s) + np.arange(-64, 64) for s in (31, 32) if (1 << s) + 64 <= nC]
    idx = np.unique(np.concatenate([sample_indices(p, nC, n)] + extra))
    got = C[torch.as_tensor(idx, device="cuda")].cpu().numpy()
    want, S = oracle.sample(case.expr, case.extents, A.cpu().numpy(), B.cpu().numpy(), idx, with_scale=True)
    bad = np.flatnonzero(~(np.abs(got - want) <= TAU64 * S))
    assert bad.size == 0, (n, idx[bad[:5]], got[bad[:5]], want[bad[:5]])
    assert not bool(torch.isnan(C).any())   # every element was written
    del C
    torch.cuda.empty_cache()


@pytest.mark.parametrize("dtype", ["bf16", "tf32", "f32"])
@pytest.mark.parametrize("cid", [1, 2, 3, 4, 5, 6, 7, 8, 18])
def test_membound_suite_full_size_tuned(dtype, cid):
    # bench.py's membound suite (BASELINE config 4), every row, tuned as the bench tunes it
    case = [c for c in tcinputs.tccg48() if c.id == cid][0]
    p, A, B, C, _ = run_tuned(case, dtype=dtype)
    check_sampled(p, case, dtype, A, B, C, seed=cid)
    assert not bool(torch.isnan(C.float()).any())


@pytest.mark.parametrize("cid", list(range(40, 49)))
def test_sd2_f32_family_full_size(cid):
    # Figs. 6/7: the SD2 CCSD(T) subset in single precision — TCCG #40-48
    # (sd_t_d2, e.g. SD2_1 = abcdef-gdab-efgc) at the suite's extents, FP32 through
    # the split-TF32 tcgen05 path, model plan and tuned plan
    case = [c for c in tcinputs.tccg48() if c.id == cid][0]
    for tune in (False, True):
        p, A, B, C, _ = run_tuned(case, dtype="f32", tune=tune)
        check_sampled(p, case, "f32", A, B, C, seed=cid)
        assert not bool(torch.isnan(C).any())


@pytest.mark.parametrize("cid", [1, 6, 9, 12, 13, 16, 18, 31, 40, 48])
def test_tccg_full_size_rank1_every_element(cid):
    # A = prod u_i[idx_i], B = prod v_i[idx_i] => C[x] = prod_ext(u or v) * prod_int <u_j, v_j>
    case = [c for c in tcinputs.tccg48() if c.id == cid][0]
    c, a, b = tcinputs.split_expr(case.expr)
    ext = case.ext
    u = tcinputs.outer_factors(a, ext, 100 + cid)
    v = tcinputs.outer_factors(b, ext, 200 + cid)
    p = tc.plan(case.expr, case.extents)
    A = torch.as_tensor(tcinputs.outer_tensor(a, u), device="cuda")
    B = torch.as_tensor(tcinputs.outer_tensor(b, v), device="cuda")
    C = torch.full((p.numel("C"),), float("nan"), dtype=torch.float64, device="cuda")
    p.execute(A, B, C)
    torch.cuda.synchronize()
    fac = {x: (u[x] if x in a else v[x]) for x in c}
    want = tcinputs.outer_tensor(c, fac)
    scale = 1.0
    for j in a:
        if j not in c:
            scale *= float(np.dot(u[j], v[j]))
    want *= scale
    got = C.cpu().numpy()
    # S[x] = sum |A B| = want (all factors positive); tau * S plus the closed form's own
    # rounding (a product of <= 8 factors: 8 ulp)
    assert np.all(np.abs(got - want) <= (TAU64 + 16 * 2.2e-16) * np.abs(want))
