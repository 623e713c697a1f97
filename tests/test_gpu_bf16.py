"""GPU parity of the BF16 tcgen05 path (kernel_bf16.cuh) through the C ABI against the CPU
oracle (dtype "bf16": inputs upcast exactly, exact sum in fp64, result rounded RNE to BF16;
DESIGN.md reading R21).

Integer data => bitwise (every partial sum is an integer below 2^24, so FP32 accumulation
is exact and both sides round the same value).  Random BF16 data => per element
|C - C_exact| <= 2^-8 |C_exact| + K 2^-23 S[x]: one BF16 ulp for the final rounding of a
perturbed value plus the FP32 accumulation bound over K products (S from the oracle).
Needs a B200: run with -m gpu."""
import numpy as np
import pytest
import torch

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build
from paper_conf_cgo_kimstkpprs19_b200.csrc_variants import BF16_VARIANTS

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


def _ext_str(ext):
    return ";".join(f"{k}:{v}" for k, v in ext.items())


def _dev_bf16(bits, pad=0):
    t = torch.from_numpy(np.ascontiguousarray(bits).view(np.int16).copy()).view(torch.bfloat16)
    if pad:
        t = torch.cat([torch.zeros(pad, dtype=torch.bfloat16), t])
    return t.cuda()


def _klen(expr, extents):
    c, a, b = tcinputs.split_expr(expr)
    ext = tcinputs.parse_extents(extents)
    k = 1
    for x in set(a) & set(b):
        k *= ext[x]
    return k


def check_bf16(expr, extents, seed=0, integer=False, alpha=1.0, beta=0.0, misalign=0, cmisalign=0,
               **plan_kw):
    p = tc.plan(expr, extents, dtype="bf16", **plan_kw)
    assert p.info()["dtype"] == "bf16"
    nA, nB, nC = p.numel("A"), p.numel("B"), p.numel("C")
    gen = tcinputs.integers_np if integer else tcinputs.uniform_np
    A, B = tcinputs.bf16_bits(gen(nA, 1000 + seed)), tcinputs.bf16_bits(gen(nB, 2000 + seed))
    C0 = tcinputs.bf16_bits(gen(nC, 3000 + seed)) if beta != 0 else None
    dA, dB = _dev_bf16(A, misalign), _dev_bf16(B, misalign)
    dC = (_dev_bf16(C0, cmisalign) if C0 is not None
          else torch.full((nC + cmisalign,), float("nan"), dtype=torch.bfloat16, device="cuda"))
    p.execute_ptr(dA.data_ptr() + 2 * misalign, dB.data_ptr() + 2 * misalign, dC.data_ptr() + 2 * cmisalign,
                  alpha, beta)
    torch.cuda.synchronize()
    got = dC[cmisalign:].cpu().view(torch.int16).numpy().view(np.uint16)
    if integer:
        want = oracle.contract(expr, extents, A, B, C=C0, alpha=alpha, beta=beta, dtype="bf16")
        assert np.array_equal(got, want), (expr, extents, np.flatnonzero(got != want)[:10])
    else:
        c64 = None if C0 is None else tcinputs.bf16_to_f64(C0)
        exact, S = oracle.contract(expr, extents, tcinputs.bf16_to_f64(A), tcinputs.bf16_to_f64(B),
                                   C=c64, alpha=alpha, beta=beta, with_scale=True)
        g = tcinputs.bf16_to_f64(got)
        tol = 2.0 ** -8 * np.abs(exact) + _klen(expr, extents) * 2.0 ** -23 * S
        bad = np.flatnonzero(~(np.abs(g - exact) <= tol))
        assert bad.size == 0, (expr, extents, bad[:10], g[bad[:3]], exact[bad[:3]])
    return p


# operand layouts: (X MN-major, Y K-major), (K, MN), (MN, MN), (K, K) and the Table-I shapes
LAYOUTS = [
    ("ab-ac-cb", "a:200;b:150;c:130"),
    ("ab-ca-bc", "a:256;b:136;c:192"),
    ("ab-ac-bc", "a:131;b:97;c:80"),
    ("ab-ca-cb", "a:128;b:64;c:72"),
    ("abcd-aebf-dfce", "a:24;b:16;c:24;d:16;e:16;f:24"),
    ("abcd-aebf-fdec", "a:16;b:24;c:8;d:40;e:24;f:9"),
    ("abcdef-gdab-efgc", "a:10;b:6;c:7;d:10;e:5;f:6;g:11"),
]


@pytest.mark.parametrize("variant", BF16_VARIANTS)
@pytest.mark.parametrize("layout", range(len(LAYOUTS)))
def test_bf16_variants_layouts(variant, layout):
    expr, ext = LAYOUTS[layout]
    check_bf16(expr, ext, seed=layout, integer=True, variant=variant)
    check_bf16(expr, ext, seed=layout, integer=False, variant=variant)


@pytest.mark.parametrize("case", tcinputs.tccg48(), ids=lambda c: f"tccg{c.id}")
def test_bf16_tccg_reduced_extents(case):
    c, a, b = tcinputs.split_expr(case.expr)
    sizes = [7, 13, 5, 11, 9, 6, 10, 3]
    ext = {x: sizes[i % len(sizes)] for i, x in enumerate(sorted(set(a + b)))}
    check_bf16(case.expr, _ext_str(ext), seed=case.id, integer=True)


def test_bf16_alpha_beta():
    e, ext = "abcd-aebf-dfce", "a:9;b:10;c:11;d:12;e:5;f:7"
    check_bf16(e, ext, seed=3, integer=True, alpha=2.0, beta=1.0)
    check_bf16(e, ext, seed=4, alpha=0.5, beta=-1.25)
    # staged 16-B epilogue (C's FVI leads m in multiples of 8), with and without beta
    e, ext = "abcdef-gdab-efgc", "a:16;b:6;c:7;d:10;e:5;f:6;g:11"
    assert tc.plan(e, ext, dtype="bf16", host_only=True).info()["vecC"] == 8
    check_bf16(e, ext, seed=5, integer=True, alpha=2.0, beta=1.0)
    check_bf16(e, ext, seed=6, alpha=0.5, beta=-1.25)
    check_bf16(e, ext, seed=7, integer=True)
    # C only 2-B aligned: the per-element epilogue runs
    check_bf16(e, ext, seed=8, integer=True, alpha=2.0, beta=1.0, cmisalign=1)
    check_bf16(e, ext, seed=9, integer=True, cmisalign=3)


def test_bf16_unaligned_pointers_and_tails():
    # 2-B aligned operands: the scalar (st.shared.u16) slot tables run
    check_bf16("ab-ac-cb", "a:64;b:64;c:64", seed=1, integer=True, misalign=1)
    check_bf16("ab-ca-bc", "a:130;b:66;c:70", seed=2, integer=True, misalign=3)
    # ragged tails in every dimension, many k-steps
    check_bf16("ab-ac-cb", "a:257;b:129;c:1000", seed=5, integer=True)
    check_bf16("C[] = A[a,b] * B[b,a]", "a:37;b:29", seed=6, integer=True)


def test_bf16_eq1_full():
    # eq. (1), all extents 16 (BASELINE config 1)
    check_bf16(tcinputs.EQ1_EXPR, tcinputs.EQ1_EXTENTS, seed=0, integer=True)
    check_bf16(tcinputs.EQ1_EXPR, tcinputs.EQ1_EXTENTS, seed=0)
