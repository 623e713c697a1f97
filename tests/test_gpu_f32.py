"""GPU parity of the FP32-storage tcgen05 paths (kernel_umma.cuh) through the C ABI against
the CPU oracle (oracle/: exact sum in fp64 of the FP32 inputs, rounded RNE to FP32).

dtype "f32" (TC_F32, FP32 as split TF32: hi*hi + hi*lo + lo*hi):
    |C - C_exact| <= 1e-5 * S[x]      (north_star's FP32 tolerance; S = sum |A||B| + |beta C|)
dtype "tf32" (TC_TF32, kind::tf32 on FP32 data; reading R30):
    |C - C_exact| <= 2^-9 * S[x] + 2^-23 |C_exact|   (each TF32 input carries <= 2^-10 relative
    error -> <= 2^-9 per product; FP32 accumulation and the final rounding are far below)
Integer data in [-3, 3] => bit-exact on both (TF32 holds them exactly, every partial sum is an
integer below 2^24, so FP32 accumulation is exact and both sides round the same value).
Needs a B200: run with -m gpu."""
import numpy as np
import pytest
import torch

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build
from paper_conf_cgo_kimstkpprs19_b200.csrc_variants import F32_VARIANTS, TF32_VARIANTS

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


def _ext_str(ext):
    return ";".join(f"{k}:{v}" for k, v in ext.items())


def _dev_f32(x, pad=0):
    t = torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32))
    if pad:
        t = torch.cat([torch.zeros(pad, dtype=torch.float32), t])
    return t.cuda()


def check_f32(expr, extents, dtype, seed=0, integer=False, alpha=1.0, beta=0.0, misalign=0,
              cmisalign=0, **plan_kw):
    p = tc.plan(expr, extents, dtype=dtype, **plan_kw)
    assert p.info()["dtype"] == dtype
    nA, nB, nC = p.numel("A"), p.numel("B"), p.numel("C")
    gen = tcinputs.integers_np if integer else tcinputs.uniform_np
    A = gen(nA, 1000 + seed).astype(np.float32)
    B = gen(nB, 2000 + seed).astype(np.float32)
    C0 = gen(nC, 3000 + seed).astype(np.float32) if beta != 0 else None
    dA, dB = _dev_f32(A, misalign), _dev_f32(B, misalign)
    dC = (_dev_f32(C0, cmisalign) if C0 is not None
          else torch.full((nC + cmisalign,), float("nan"), dtype=torch.float32, device="cuda"))
    p.execute_ptr(dA.data_ptr() + 4 * misalign, dB.data_ptr() + 4 * misalign, dC.data_ptr() + 4 * cmisalign,
                  alpha, beta)
    torch.cuda.synchronize()
    got = dC[cmisalign:].cpu().numpy()
    if integer:
        want = oracle.contract(expr, extents, A, B, C=C0, alpha=alpha, beta=beta, dtype="f32")
        assert np.array_equal(got, want), (expr, extents, np.flatnonzero(got != want)[:10])
        return p, 0.0
    exact, S = oracle.contract(expr, extents, A.astype(np.float64), B.astype(np.float64),
                               C=None if C0 is None else C0.astype(np.float64), alpha=alpha, beta=beta,
                               with_scale=True)
    g = got.astype(np.float64)
    if dtype == "f32":
        tol = 1e-5 * S
    else:
        tol = 2.0 ** -9 * S + 2.0 ** -23 * np.abs(exact)
    bad = np.flatnonzero(~(np.abs(g - exact) <= tol))
    assert bad.size == 0, (expr, extents, dtype, bad[:10], g[bad[:3]], exact[bad[:3]])
    return p, float(np.max(np.abs(g - exact) / np.maximum(S, 1e-300)))


LAYOUTS = [
    ("ab-ac-cb", "a:200;b:150;c:130"),
    ("ab-ca-bc", "a:256;b:136;c:192"),
    ("ab-ac-bc", "a:131;b:97;c:80"),
    ("ab-ca-cb", "a:128;b:64;c:72"),
    ("abcd-aebf-dfce", "a:24;b:16;c:24;d:16;e:16;f:24"),
    ("abcd-aebf-fdec", "a:16;b:24;c:8;d:40;e:24;f:9"),
    ("abcdef-gdab-efgc", "a:10;b:6;c:7;d:10;e:5;f:6;g:11"),
]


@pytest.mark.parametrize("variant", TF32_VARIANTS + F32_VARIANTS)
@pytest.mark.parametrize("layout", range(len(LAYOUTS)))
def test_f32_variants_layouts(variant, layout):
    dtype = "tf32" if variant in TF32_VARIANTS else "f32"
    expr, ext = LAYOUTS[layout]
    check_f32(expr, ext, dtype, seed=layout, integer=True, variant=variant)
    check_f32(expr, ext, dtype, seed=layout, integer=False, variant=variant)


@pytest.mark.parametrize("dtype", ["f32", "tf32"])
@pytest.mark.parametrize("case", tcinputs.tccg48(), ids=lambda c: f"tccg{c.id}")
def test_f32_tccg_reduced_extents(case, dtype):
    c, a, b = tcinputs.split_expr(case.expr)
    sizes = [7, 13, 5, 11, 9, 6, 10, 3]
    ext = {x: sizes[i % len(sizes)] for i, x in enumerate(sorted(set(a + b)))}
    check_f32(case.expr, _ext_str(ext), dtype, seed=case.id, integer=True)
    check_f32(case.expr, _ext_str(ext), dtype, seed=case.id)


@pytest.mark.parametrize("dtype", ["f32", "tf32"])
def test_f32_alpha_beta_alignment_tails(dtype):
    e, ext = "abcd-aebf-dfce", "a:9;b:10;c:11;d:12;e:5;f:7"
    check_f32(e, ext, dtype, seed=3, integer=True, alpha=2.0, beta=1.0)
    check_f32(e, ext, dtype, seed=4, alpha=0.5, beta=-1.25)
    e, ext = "abcdef-gdab-efgc", "a:16;b:6;c:7;d:10;e:5;f:6;g:11"
    assert tc.plan(e, ext, dtype=dtype, host_only=True).info()["vecC"] == 8
    check_f32(e, ext, dtype, seed=5, integer=True, alpha=2.0, beta=1.0)
    check_f32(e, ext, dtype, seed=6, alpha=0.5, beta=-1.25)
    check_f32(e, ext, dtype, seed=8, integer=True, alpha=2.0, beta=1.0, cmisalign=1)
    # 4-B aligned operands: the scalar slot tables run
    check_f32("ab-ac-cb", "a:64;b:64;c:64", dtype, seed=1, integer=True, misalign=1)
    check_f32("ab-ca-bc", "a:130;b:66;c:70", dtype, seed=2, integer=True, misalign=3)
    # ragged tails, many k-steps, a scalar result
    check_f32("ab-ac-cb", "a:257;b:129;c:1000", dtype, seed=5, integer=True)
    check_f32("ab-ac-cb", "a:257;b:129;c:1000", dtype, seed=5)
    check_f32("C[] = A[a,b] * B[b,a]", "a:37;b:29", dtype, seed=6, integer=True)


def test_f32_split_is_more_accurate_than_tf32():
    # the split product must beat plain TF32 by orders of magnitude on random data
    e, ext = "abcd-aebf-dfce", "a:24;b:16;c:24;d:16;e:16;f:24"
    _, err32 = check_f32(e, ext, "f32", seed=11)
    _, errtf = check_f32(e, ext, "tf32", seed=11)
    assert err32 < 3e-6 and errtf > 30 * err32, (err32, errtf)


@pytest.mark.parametrize("cid", [1, 6, 8, 18])
def test_f32_memory_bound_full_size_sampled(cid):
    # BASELINE config 4: the memory-bound TCCG cases at full size, FP32; sampled elements
    case = [c for c in tcinputs.tccg48() if c.id == cid][0]
    p = tc.plan(case.expr, case.extents, dtype="f32")
    A = tcinputs.uniform(p.numel("A"), 1000 + cid, device="cuda").float()
    B = tcinputs.uniform(p.numel("B"), 2000 + cid, device="cuda").float()
    C = torch.full((p.numel("C"),), float("nan"), dtype=torch.float32, device="cuda")
    p.execute(A, B, C)
    torch.cuda.synchronize()
    rng = np.random.default_rng(cid)
    n = p.numel("C")
    idx = np.unique(np.concatenate([rng.integers(0, n, 3000), np.arange(64), np.arange(n - 64, n)]))
    want, S = oracle.sample(case.expr, case.extents, A.cpu().numpy().astype(np.float64),
                            B.cpu().numpy().astype(np.float64), idx, with_scale=True)
    got = C.cpu().numpy()[idx].astype(np.float64)
    assert np.all(np.abs(got - want) <= 1e-5 * S)


# C's FVI as an inner m digit (the X operand's FVI leads m): the CTA-wide staged epilogue
# (kernel_umma.cuh, cs0 > 1) with 16-B runs along C's FVI, full and partial tiles, beta
TRANSPOSED = [
    ("abcde-efbad-cf", "a:16;b:3;c:24;d:5;e:16;f:12"),
    ("abcde-efcad-bf", "a:24;b:10;c:3;d:2;e:32;f:9"),
    ("abcd-dbea-ec", "a:40;b:3;c:24;d:16;e:24"),
    ("abcd-deca-be", "a:8;b:20;c:3;d:72;e:36"),
    ("abc-bda-dc", "a:48;b:40;c:24;d:30"),
]


@pytest.mark.parametrize("dtype", ["f32", "tf32", "bf16"])
@pytest.mark.parametrize("layout", range(len(TRANSPOSED)))
def test_umma_inner_fvi_epilogue(dtype, layout):
    expr, ext = TRANSPOSED[layout]
    info = tc.plan(expr, ext, dtype=dtype, host_only=True, morder="X").info()
    assert info["vecC"] == 8 and info["cs0"] > 1, info
    if dtype == "bf16":
        from tests.test_gpu_bf16 import check_bf16
        check_bf16(expr, ext, seed=layout, integer=True, morder="X")
        check_bf16(expr, ext, seed=layout, integer=True, alpha=2.0, beta=1.0, morder="X")
        check_bf16(expr, ext, seed=layout, morder="X")
    else:
        check_f32(expr, ext, dtype, seed=layout, integer=True, morder="X")
        check_f32(expr, ext, dtype, seed=layout, integer=True, alpha=2.0, beta=1.0, morder="X")
        check_f32(expr, ext, dtype, seed=layout, alpha=0.5, beta=-1.25, morder="X")


@pytest.mark.parametrize("dtype", ["f32", "tf32", "bf16"])
@pytest.mark.parametrize("expr,ext", [("hij-hik-hkj", "h:3;i:130;j:64;k:70"),
                                      ("abcd-aebd-ecd", "a:24;b:6;c:40;d:3;e:50"),
                                      ("abc-ab-cb", "a:30;b:4;c:50"), ("ab-ab-ab", "a:5;b:7")])
def test_umma_batch_indices(dtype, expr, ext):
    if dtype == "bf16":
        from tests.test_gpu_bf16 import check_bf16
        check_bf16(expr, ext, seed=1, integer=True)
        check_bf16(expr, ext, seed=2, integer=True, alpha=2.0, beta=1.0)
        check_bf16(expr, ext, seed=3)
    else:
        check_f32(expr, ext, dtype, seed=1, integer=True)
        check_f32(expr, ext, dtype, seed=2, integer=True, alpha=2.0, beta=1.0)
        check_f32(expr, ext, dtype, seed=3)
