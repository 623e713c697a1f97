"""Full-size parity: every TCCG-48 contraction at the benchmark extents,
in the exact launch configuration bench.py times (same plan, same seeded device inputs),
checked against the CPU oracle on sampled outputs (random + first + last elements), and
against the rank-1 closed form on EVERY output element for a subset.  Needs a B200."""
import numpy as np
import pytest
import torch

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build

pytestmark = pytest.mark.gpu
TAU64 = 1e-12


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


@pytest.mark.parametrize("case", tcinputs.tccg48(), ids=lambda c: f"tccg{c.id}")
def test_tccg_full_size_sampled(case):
    p = tc.plan(case.expr, case.extents)
    A = tcinputs.uniform(p.numel("A"), 1000 + case.id, device="cuda")
    B = tcinputs.uniform(p.numel("B"), 2000 + case.id, device="cuda")
    C = torch.full((p.numel("C"),), float("nan"), dtype=torch.float64, device="cuda")
    p.execute(A, B, C)
    torch.cuda.synchronize()
    n = C.numel()
    rng = np.random.default_rng(case.id)
    idx = np.unique(np.concatenate([rng.integers(0, n, 1500), np.arange(min(n, 256)),
                                    np.arange(max(0, n - 256), n)]))
    got = C[torch.as_tensor(idx, device="cuda")].cpu().numpy()
    want, S = oracle.sample(case.expr, case.extents, A.cpu().numpy(), B.cpu().numpy(), idx,
                            with_scale=True)
    bad = np.flatnonzero(~(np.abs(got - want) <= TAU64 * S))
    assert bad.size == 0, (case.id, idx[bad[:5]], got[bad[:5]], want[bad[:5]])
    assert torch.isfinite(C).all()          # every element was written


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


@pytest.mark.parametrize("n,expr", [(48, "abcdef-gdab-efgc"), (40, "abcdef-dega-gfbc")])
def test_ccsdt_max_size_sampled(n, expr):
    # BASELINE config 3 at its largest extent: |C| = 48^6 = 1.2e10 FP64 elements (97.8 GB) —
    # past 2^31 elements, so every 64-bit offset path of the tables and the epilogue runs
    case = tcinputs.ccsdt(n, expr, 100 + n)
    p = tc.plan(case.expr, case.extents)
    A = tcinputs.uniform(p.numel("A"), 1000 + case.id, device="cuda")
    B = tcinputs.uniform(p.numel("B"), 2000 + case.id, device="cuda")
    C = torch.full((p.numel("C"),), float("nan"), dtype=torch.float64, device="cuda")
    p.execute(A, B, C)
    torch.cuda.synchronize()
    nC = C.numel()
    rng = np.random.default_rng(n)
    idx = np.unique(np.concatenate([rng.integers(0, nC, 2000), np.arange(128), np.arange(nC - 128, nC),
                                    (np.int64(1) << 31) + np.arange(-64, 64)]))
    got = C[torch.as_tensor(idx, device="cuda")].cpu().numpy()
    want, S = oracle.sample(case.expr, case.extents, A.cpu().numpy(), B.cpu().numpy(), idx,
                            with_scale=True)
    bad = np.flatnonzero(~(np.abs(got - want) <= TAU64 * S))
    assert bad.size == 0, (n, idx[bad[:5]], got[bad[:5]], want[bad[:5]])
    assert not bool(torch.isnan(C).any())   # every element was written
    del C
    torch.cuda.empty_cache()


@pytest.mark.parametrize("cid", [1, 8, 12, 18, 30, 33, 40])
def test_tuned_plans_as_bench_times_them(cid):
    # bench.py times tc_plan_tuned plans (top-8 variants measured); check those, sampled
    case = [c for c in tcinputs.tccg48() if c.id == cid][0]
    p = tc.plan(case.expr, case.extents)
    A = tcinputs.uniform(p.numel("A"), 1000 + case.id, device="cuda")
    B = tcinputs.uniform(p.numel("B"), 2000 + case.id, device="cuda")
    C = torch.empty(p.numel("C"), dtype=torch.float64, device="cuda")
    p = p.tuned(A, B, C, topk=8, reps=1)
    C.fill_(float("nan"))
    p.execute(A, B, C)
    torch.cuda.synchronize()
    n = C.numel()
    idx = np.unique(np.concatenate([np.random.default_rng(cid).integers(0, n, 1500), np.arange(64),
                                    np.arange(n - 64, n)]))
    got = C[torch.as_tensor(idx, device="cuda")].cpu().numpy()
    want, S = oracle.sample(case.expr, case.extents, A.cpu().numpy(), B.cpu().numpy(), idx, with_scale=True)
    assert np.all(np.abs(got - want) <= TAU64 * S), (cid, p.info()["variant"])
    assert torch.isfinite(C).all()


@pytest.mark.parametrize("dtype", ["bf16", "tf32", "f32"])
@pytest.mark.parametrize("cid", [1, 4, 6, 7])
def test_membound_suite_full_size_sampled(dtype, cid):
    # BASELINE config 4 at full size in the bench's launch configuration (tuned plan)
    case = [c for c in tcinputs.tccg48() if c.id == cid][0]
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    p = tc.plan(case.expr, case.extents, dtype=dtype)
    A = tcinputs.uniform(p.numel("A"), 1000 + cid, device="cuda").to(tdt)
    B = tcinputs.uniform(p.numel("B"), 2000 + cid, device="cuda").to(tdt)
    C = torch.empty(p.numel("C"), dtype=tdt, device="cuda")
    p = p.tuned(A, B, C, topk=8, reps=1)
    C.fill_(float("nan"))
    p.execute(A, B, C)
    torch.cuda.synchronize()
    n = C.numel()
    idx = np.unique(np.concatenate([np.random.default_rng(cid).integers(0, n, 2000), np.arange(64),
                                    np.arange(n - 64, n)]))
    got = C[torch.as_tensor(idx, device="cuda")].float().cpu().numpy().astype(np.float64)
    exact, S = oracle.sample(case.expr, case.extents, A.double().cpu().numpy(), B.double().cpu().numpy(),
                             idx, with_scale=True)
    K = p.flops / 2 / n
    if dtype == "f32":
        tol = 1e-5 * S
    elif dtype == "tf32":
        tol = 2.0 ** -9 * S + 2.0 ** -23 * np.abs(exact)
    else:   # DESIGN R21 / test_gpu_bf16: one BF16 ulp of the result + FP32 accumulation
        tol = 2.0 ** -8 * np.abs(exact) + K * 2.0 ** -23 * S
    bad = np.flatnonzero(~(np.abs(got - exact) <= tol))
    assert bad.size == 0, (cid, dtype, idx[bad[:5]], got[bad[:5]], exact[bad[:5]])
