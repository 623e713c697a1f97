"""GPU parity: libtc's CUDA path (through the C ABI) against the CPU oracle, element by
element, on the same seeded inputs (tcinputs).  Integer data => bitwise; random data =>
|C - C_ref| <= tau * S[x] with S[x] = |alpha| sum|A*B| + |beta||C_in| (tau = 1e-12, FP64).
Needs a B200: run with -m gpu."""
import numpy as np
import pytest
import torch

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build
from paper_conf_cgo_kimstkpprs19_b200.csrc_variants import F64_VARIANTS, STG_VARIANTS
from tests.layouts import PRIME_EXT, layouts_one_contraction, layouts_two_contractions

pytestmark = pytest.mark.gpu
TAU64 = 1e-12


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


def _ext_str(ext):
    return ";".join(f"{k}:{v}" for k, v in ext.items())


def run_gpu(p, A, B, C0=None, alpha=1.0, beta=0.0):
    dA = torch.as_tensor(np.ascontiguousarray(A), device="cuda")
    dB = torch.as_tensor(np.ascontiguousarray(B), device="cuda")
    n = p.numel("C")
    dC = (torch.as_tensor(np.ascontiguousarray(C0), device="cuda").clone() if C0 is not None
          else torch.full((n,), float("nan"), dtype=torch.float64, device="cuda"))
    p.execute(dA, dB, dC, alpha, beta)
    torch.cuda.synchronize()
    return dC.cpu().numpy()


def check_case(expr, extents, seed=0, integer=False, alpha=1.0, beta=0.0, **plan_kw):
    c, a, b = (tcinputs.split_expr(expr) if "[" not in expr else (None, None, None))
    p = tc.plan(expr, extents, **plan_kw)
    nA, nB, nC = p.numel("A"), p.numel("B"), p.numel("C")
    gen = tcinputs.integers_np if integer else tcinputs.uniform_np
    A, B = gen(nA, 1000 + seed), gen(nB, 2000 + seed)
    C0 = gen(nC, 3000 + seed) if beta != 0 else None
    got = run_gpu(p, A, B, C0, alpha, beta)
    want, S = oracle.contract(expr, extents, A, B, C=C0, alpha=alpha, beta=beta, with_scale=True)
    if integer:
        assert np.array_equal(got, want), (expr, extents, np.flatnonzero(got != want)[:10])
    else:
        err = np.abs(got - want)
        bad = np.flatnonzero(~(err <= TAU64 * S))
        assert bad.size == 0, (expr, extents, bad[:10], got[bad[:3]], want[bad[:3]])
    return p


def test_eq1_worked_example():
    # eq. (1), all extents 16 (BASELINE config 1)
    check_case(tcinputs.EQ1_EXPR, tcinputs.EQ1_EXTENTS, seed=0)
    check_case(tcinputs.EQ1_EXPR, tcinputs.EQ1_EXTENTS, seed=0, integer=True)
    check_case("C[a,b,c,d] = A[a,e,b,f] * B[d,f,c,e]", tcinputs.EQ1_EXTENTS, seed=1)


@pytest.mark.parametrize("family", ["one", "two"])
def test_all_layouts_p_l27_bitwise(family):
    exprs = layouts_one_contraction() if family == "one" else layouts_two_contractions()
    for n, expr in enumerate(exprs):
        c, a, b = tcinputs.split_expr(expr)
        ext = {x: PRIME_EXT[x] for x in sorted(set(a + b))}
        check_case(expr, _ext_str(ext), seed=n, integer=True)


@pytest.mark.parametrize("case", tcinputs.tccg48(), ids=lambda c: f"tccg{c.id}")
def test_tccg_reduced_extents(case):
    # the suite's index structure at extents small enough for the full oracle, spanning
    # several tiles with ragged tails (odd / prime extents)
    c, a, b = tcinputs.split_expr(case.expr)
    sizes = [7, 13, 5, 11, 9, 6, 10, 3]
    ext = {x: sizes[i % len(sizes)] for i, x in enumerate(sorted(set(a + b)))}
    check_case(case.expr, _ext_str(ext), seed=case.id)
    check_case(case.expr, _ext_str(ext), seed=case.id, integer=True)


def test_alpha_beta_and_nan_c():
    e = "abcd-aebf-dfce"
    ext = "a:9;b:10;c:11;d:12;e:5;f:7"
    check_case(e, ext, seed=3, alpha=0.5, beta=-1.25)
    check_case(e, ext, seed=4, integer=True, alpha=2.0, beta=1.0)
    # beta == 0 with NaN in C: run_gpu pre-fills C with NaN
    check_case(e, ext, seed=5, integer=True, alpha=1.0, beta=0.0)


@pytest.mark.parametrize("tma", [True, False])
@pytest.mark.parametrize("variant", F64_VARIANTS)
def test_every_kernel_variant(variant, tma):
    # both epilogues: TMA box store (cp.async.bulk.tensor) and predicated direct stores
    check_case("abcdef-gdab-efgc", "a:10;b:6;c:7;d:10;e:5;f:6;g:11", seed=variant, integer=True,
               variant=variant, tma=tma)
    check_case("abcd-aebf-dfce", "a:18;b:9;c:13;d:20;e:19;f:3", seed=variant, variant=variant, tma=tma)
    check_case("abcd-aebf-fdec", "a:16;b:24;c:8;d:40;e:24;f:9", seed=variant, variant=variant, tma=tma)


@pytest.mark.parametrize("variant", STG_VARIANTS)
def test_staged_epilogue_alpha_beta(variant):
    # the producers' drain applies alpha / beta: 16-B pairs (C's FVI tile and extent even)
    # and the scalar path (odd FVI extent), partial tiles on every side, several tiles per CTA
    check_case("abcd-aebf-dfce", "a:36;b:7;c:9;d:30;e:6;f:5", seed=variant, alpha=0.5, beta=-1.25,
               variant=variant)
    check_case("abcd-aebf-dfce", "a:35;b:7;c:9;d:30;e:6;f:5", seed=variant, integer=True, alpha=2.0,
               beta=1.0, variant=variant)
    check_case("abcdef-gdab-efgc", "a:24;b:6;c:7;d:10;e:5;f:6;g:24", seed=variant, integer=True,
               variant=variant)


def test_paper_cost_mode_runs():
    check_case("abcd-aebf-dfce", "a:24;b:20;c:16;d:30;e:12;f:10", seed=7, cost="paper")


def test_forced_fig3_tiles_run():
    check_case("abcd-aebf-dfce", tcinputs.EQ1_EXTENTS, seed=8, integer=True,
               force_tiles="a:16;e:1;b:4;f:16;d:4;c:1")


def test_degenerate_shapes():
    check_case("abcd-ab-cd", "a:3;b:5;c:7;d:2", seed=1)                 # outer product
    check_case("C[] = A[a,b] * B[b,a]", "a:37;b:29", seed=2)            # scalar C
    check_case("abcd-aebf-dfce", "a:1;b:5;c:1;d:7;e:1;f:9", seed=3)     # extent-1 indices
    check_case("ab-ac-cb", "a:1;b:1;c:1", seed=4)                       # one element
    check_case("ab-ac-cb", "a:257;b:129;c:65", seed=5)                  # odd tails
    check_case("ab-ca-bc", "a:100;b:300;c:1000", seed=6)                # transposed GEMM


def test_unaligned_pointers_use_scalar_loads():
    p = tc.plan("ab-ac-cb", "a:64;b:64;c:64")
    A = tcinputs.integers_np(64 * 64, 1)
    B = tcinputs.integers_np(64 * 64, 2)
    dA = torch.zeros(64 * 64 + 1, dtype=torch.float64, device="cuda")
    dB = torch.zeros(64 * 64 + 1, dtype=torch.float64, device="cuda")
    dA[1:] = torch.as_tensor(A, device="cuda")
    dB[1:] = torch.as_tensor(B, device="cuda")
    dC = torch.zeros(64 * 64, dtype=torch.float64, device="cuda")
    p.execute_ptr(dA.data_ptr() + 8, dB.data_ptr() + 8, dC.data_ptr())
    torch.cuda.synchronize()
    assert np.array_equal(dC.cpu().numpy(), oracle.contract("ab-ac-cb", "a:64;b:64;c:64", A, B))


def test_restricted_slabs_reassemble():
    expr, ext = "abcdef-gdab-efgc", "a:8;b:5;c:6;d:7;e:4;f:9;g:10"
    p = tc.plan(expr, ext)
    A = tcinputs.integers_np(p.numel("A"), 1)
    B = tcinputs.integers_np(p.numel("B"), 2)
    full = oracle.contract(expr, ext, A, B)
    dA = torch.as_tensor(A, device="cuda")
    dB = torch.as_tensor(B, device="cuda")
    dC = torch.full((p.numel("C"),), float("nan"), dtype=torch.float64, device="cuda")
    for lo, ln in [(0, 4), (4, 3), (7, 2)]:           # C-slab sharding on f (8(e))
        p.restrict("f", lo, ln).execute(dA, dB, dC)
    torch.cuda.synchronize()
    assert np.array_equal(dC.cpu().numpy(), full)
    # split-K over g: partial sums add up to the full result
    acc = torch.zeros_like(dC)
    for lo, ln in [(0, 3), (3, 7)]:
        part = torch.zeros_like(dC)
        p.restrict("g", lo, ln).execute(dA, dB, part)
        acc += part
    torch.cuda.synchronize()
    assert np.array_equal(acc.cpu().numpy(), full)
    # compact C slab (TC_SLAB_C)
    sub = p.restrict("f", 3, 4, tc.SLAB_C)
    dCs = torch.zeros(sub.numel("C"), dtype=torch.float64, device="cuda")
    sub.execute(dA, dB, dCs)
    torch.cuda.synchronize()
    per_f = p.numel("C") // 9
    assert np.array_equal(dCs.cpu().numpy(), full[3 * per_f:7 * per_f])


def test_overlap_and_device_errors():
    p = tc.plan("ab-ac-cb", "a:8;b:8;c:8")
    A = torch.zeros(64, dtype=torch.float64, device="cuda")
    with pytest.raises(tc.TcError) as e:
        p.execute_ptr(A.data_ptr(), A.data_ptr(), A.data_ptr())
    assert e.value.status == "TC_ERR_INVALID_ARG"
    with pytest.raises(tc.TcError):
        p.execute_ptr(0, A.data_ptr(), A.data_ptr())


def test_execute_host_end_to_end():
    expr, ext = "abcd-dbea-ec", "a:20;b:18;c:6;d:22;e:14"
    p = tc.plan(expr, ext)
    A = torch.as_tensor(tcinputs.uniform_np(p.numel("A"), 1)).pin_memory()
    B = torch.as_tensor(tcinputs.uniform_np(p.numel("B"), 2)).pin_memory()
    C = torch.zeros(p.numel("C"), dtype=torch.float64).pin_memory()
    ws = torch.empty(p.workspace_bytes() // 8 + 1, dtype=torch.float64, device="cuda")
    p.execute_host(A, B, C, ws)
    want, S = oracle.contract(expr, ext, A.numpy(), B.numpy(), with_scale=True)
    assert np.all(np.abs(C.numpy() - want) <= TAU64 * S)


def test_measured_tuning_returns_a_correct_plan():
    # tc_plan_tuned: times the top-k variants' best configs on the
    # caller's tensors and returns the fastest as a new plan; the result must stay exact
    expr, ext = "abcdef-gdab-efgc", "a:24;b:16;c:16;d:24;e:16;f:16;g:24"
    p = tc.plan(expr, ext)
    A = tcinputs.integers_np(p.numel("A"), 11)
    B = tcinputs.integers_np(p.numel("B"), 12)
    dA = torch.as_tensor(A, device="cuda")
    dB = torch.as_tensor(B, device="cuda")
    dC = torch.empty(p.numel("C"), dtype=torch.float64, device="cuda")
    t = p.tuned(dA, dB, dC, topk=3, reps=2)
    info = t.info()
    assert len(info["stats"]["tuned"]) == 3
    assert info["variant"] in [v for v, _ in info["stats"]["tuned"]]
    dC.fill_(float("nan"))
    t.execute(dA, dB, dC)
    torch.cuda.synchronize()
    assert np.array_equal(dC.cpu().numpy(), oracle.contract(expr, ext, A, B))
    with pytest.raises(tc.TcError):
        p.tuned(dA, dB, dC, topk=0)


# Batch (Hadamard) indices (R31): grid y walks the batch slabs
BATCH = [
    ("hij-hik-hkj", "h:3;i:40;j:50;k:60"),          # batched GEMM, batch index fastest
    ("ijh-ikh-kjh", "h:7;i:64;j:72;k:32"),          # batch index slowest
    ("abcd-aebd-ecd", "a:24;b:6;c:40;d:3;e:50"),
    ("abcd-dbea-ecb", "a:16;b:3;c:24;d:9;e:20"),    # batch in the middle of every tensor
    ("ab-ab-ab", "a:5;b:7"),                        # pure Hadamard product
    ("abc-ab-cb", "a:30;b:4;c:50"),                 # batched outer product
    ("C[h,g,i] = A[g,k,h] * B[k,i,g,h]", "h:2;g:3;i:40;k:50"),
]


@pytest.mark.parametrize("expr,ext", BATCH)
def test_batch_indices(expr, ext):
    check_case(expr, ext, seed=7, integer=True)
    check_case(expr, ext, seed=8)
    check_case(expr, ext, seed=9, alpha=0.5, beta=-1.5)
    for v in (2, 13, 19):                           # direct, staged and wide warp tiles
        check_case(expr, ext, seed=10, integer=True, variant=v)


def test_cached_plan_executes_and_is_shared():
    # NEXT-1: tc_plan_cached returns the same plan for the same arguments; it runs like any plan
    tc.plan_cache_clear()
    e, x = "abcd-aebf-dfce", "a:24;b:16;c:24;d:16;e:16;f:24"
    p1 = tc.plan_cached(e, x)
    p2 = tc.plan_cached(e, x)
    assert p1.handle.value == p2.handle.value and tc.plan_cache_size() == 1
    A = tcinputs.integers_np(p1.numel("A"), 5)
    B = tcinputs.integers_np(p1.numel("B"), 6)
    got = run_gpu(p2, A, B)
    assert np.array_equal(got, oracle.contract(e, x, A, B))
    del p1
    tc.plan_cache_clear()
    assert np.array_equal(run_gpu(p2, A, B), got)   # the caller's reference outlives the cache


def test_tma_plan_survives_a_later_plain_plan_on_the_same_kernel():
    """The dynamic-smem attribute belongs to the kernel instance that many plans share: a TMA
    epilogue plan, then a plan WITHOUT it on the same variant and layouts, then the TMA plan
    again must still launch and be right (the later plan used to shrink the limit)."""
    expr, ext = "abcd-aebf-dfce", "a:16;b:16;c:16;d:16;e:16;f:16"
    A, B = tcinputs.uniform_np(16 ** 4, 11), tcinputs.uniform_np(16 ** 4, 12)
    want, S = oracle.contract(expr, ext, A, B, with_scale=True)
    for v in (3, 0):
        p_tma = tc.plan(expr, ext, variant=v, tma=True)
        p_plain = tc.plan(expr, ext, variant=v, tma=False)
        for p in (p_tma, p_plain, p_tma):
            got = run_gpu(p, A, B)
            assert np.all(np.abs(got - want) <= TAU64 * S), (v, p is p_tma)
