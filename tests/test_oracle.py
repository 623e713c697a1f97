"""Pins of the CPU oracle against things other than itself (SURVEY 8(c) "What pins each part").

Every test here is CPU-only.  The oracle (oracle/tc_oracle.c) is compared with:
  * the validation rules table (tests/golden/validation_rules.json);
  * brute-force TTGT on all 864 + 72 layouts of P:L27, bitwise, integer data;
  * torch.einsum (fp64) on random data, within tau;
  * GEMM special cases (ab-ac-cb and transposes) against numpy matmul / a triple loop;
  * the rank-1 closed form, constant inputs, delta inputs (permutation of A);
  * linearity, alpha/beta algebra, NaN in C with beta == 0;
  * relabelling invariance, operand swap and output permutation (bitwise, integer data);
  * slab consistency (range pieces concatenate bitwise) and sample == range;
  * its own Neumaier mode against math.fsum, and bf16/f32 output rounding properties.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
import tcinputs
from tests.layouts import PRIME_EXT, layouts_one_contraction, layouts_two_contractions
from tests.ttgt import einsum_ref, ttgt

HERE = os.path.dirname(os.path.abspath(__file__))
TAU64 = 1e-12


def _ext_str(ext, idx):
    return ";".join(f"{c}:{ext[c]}" for c in sorted(set(idx)))


def test_validation_rules_golden():
    rules = json.load(open(os.path.join(HERE, "golden", "validation_rules.json")))["rules"]
    for expr, extents, want in rules:
        assert oracle.check(expr, extents) == want, (expr, extents)


def test_layout_counts_p_l27():
    # 3! x 3! x 4! (printed "846", product 864) and 72.
    one, two = layouts_one_contraction(), layouts_two_contractions()
    assert len(one) == len(set(one)) == 864
    assert len(two) == len(set(two)) == 72


@pytest.mark.parametrize("family", ["one", "two"])
def test_ttgt_all_layouts_bitwise(family):
    exprs = layouts_one_contraction() if family == "one" else layouts_two_contractions()
    for n, expr in enumerate(exprs):
        c, a, b = tcinputs.split_expr(expr)
        ext = {x: PRIME_EXT[x] for x in set(a + b)}
        A = tcinputs.integers_np(tcinputs.numel(a, ext), 10 + n)
        B = tcinputs.integers_np(tcinputs.numel(b, ext), 20 + n)
        got = oracle.contract(expr, _ext_str(ext, a + b), A, B)
        want = ttgt(c, a, b, ext, A, B)
        assert np.array_equal(got, want), expr


def test_eq1_worked_example_ttgt_and_einsum():
    # eq. (1): C[a,b,c,d] = A[a,e,b,f] * B[d,f,c,e]; distinct extents.
    ext = {"a": 3, "b": 4, "c": 5, "d": 2, "e": 6, "f": 7}
    es = _ext_str(ext, "abcdef")
    A = tcinputs.integers_np(3 * 6 * 4 * 7, 1)
    B = tcinputs.integers_np(2 * 7 * 5 * 6, 2)
    got = oracle.contract("abcd-aebf-dfce", es, A, B)
    assert np.array_equal(got, ttgt("abcd", "aebf", "dfce", ext, A, B))
    # bracket grammar gives the identical result
    got2 = oracle.contract("C[a,b,c,d] = A[a,e,b,f] * B[d,f,c,e]", es, A, B)
    assert np.array_equal(got, got2)
    # explicit element: C[1,2,3,1] = sum_{e,f} A[1,e,2,f] B[1,f,3,e]
    An = A.reshape(7, 4, 6, 3)   # axes f, b, e, a
    Bn = B.reshape(6, 5, 7, 2)   # axes e, c, f, d
    s = sum(An[f, 2, e, 1] * Bn[e, 3, f, 1] for e in range(6) for f in range(7))
    Cn = got.reshape(2, 5, 4, 3)  # axes d, c, b, a
    assert Cn[1, 3, 2, 1] == s


@pytest.mark.parametrize("case", [c for c in tcinputs.tccg48()], ids=lambda c: f"tccg{c.id}")
def test_tccg_tiny_vs_einsum(case):
    c, a, b = tcinputs.split_expr(case.expr)
    primes = [2, 3, 5, 2, 3, 4, 3, 2]
    ext = {x: primes[i % len(primes)] for i, x in enumerate(sorted(set(a + b)))}
    A = tcinputs.uniform_np(tcinputs.numel(a, ext), 1000 + case.id)
    B = tcinputs.uniform_np(tcinputs.numel(b, ext), 2000 + case.id)
    got, S = oracle.contract(case.expr, _ext_str(ext, a + b), A, B, with_scale=True)
    want = einsum_ref(c, a, b, ext, A, B)
    assert np.all(np.abs(got - want) <= TAU64 * S)
    Ai = tcinputs.integers_np(A.size, 7)
    Bi = tcinputs.integers_np(B.size, 8)
    assert np.array_equal(oracle.contract(case.expr, _ext_str(ext, a + b), Ai, Bi),
                          ttgt(c, a, b, ext, Ai, Bi))


@pytest.mark.parametrize("expr", ["ab-ac-cb", "ab-ca-cb", "ab-ac-bc", "ab-ca-bc"])
def test_gemm_special_cases(expr):
    # column-major C(a,b) = sum_c A(.)B(.): the four GEMM transposition cases.
    ext = {"a": 7, "b": 5, "c": 9}
    c, a, b = tcinputs.split_expr(expr)
    A = tcinputs.uniform_np(63, 3)
    B = tcinputs.uniform_np(45, 4)
    # column-major matrices
    MA = A.reshape(ext[a[1]], ext[a[0]]).T      # rows = a[0]
    MB = B.reshape(ext[b[1]], ext[b[0]]).T
    if a[0] != "a":
        MA = MA.T                               # now rows = a, cols = c
    if b[0] != "c":
        MB = MB.T                               # now rows = c, cols = b
    want = (MA @ MB).T.reshape(-1)              # column-major flatten of C(a, b)
    got, S = oracle.contract(expr, _ext_str(ext, "abc"), A, B, with_scale=True)
    assert np.all(np.abs(got - want) <= TAU64 * S)
    # textbook triple loop, integer data, bitwise
    Ai, Bi = tcinputs.integers_np(63, 5), tcinputs.integers_np(45, 6)
    MAi = Ai.reshape(ext[a[1]], ext[a[0]]).T
    MBi = Bi.reshape(ext[b[1]], ext[b[0]]).T
    if a[0] != "a":
        MAi = MAi.T
    if b[0] != "c":
        MBi = MBi.T
    ref = np.zeros((7, 5))
    for i in range(7):
        for j in range(5):
            for k in range(9):
                ref[i, j] += MAi[i, k] * MBi[k, j]
    assert np.array_equal(oracle.contract(expr, _ext_str(ext, "abc"), Ai, Bi), ref.T.reshape(-1))


@pytest.mark.parametrize("expr,ext", [
    ("abcd-aebf-dfce", {c: 6 for c in "abcdef"}),
    ("abcdef-gdab-efgc", {"a": 5, "b": 4, "c": 3, "d": 5, "e": 4, "f": 3, "g": 6}),
    ("abcde-efbad-cf", {"a": 4, "b": 3, "c": 2, "d": 3, "e": 4, "f": 3}),
    ("abc-adec-ebd", {"a": 5, "b": 4, "c": 3, "d": 5, "e": 4}),
])
def test_rank1_closed_form(expr, ext):
    # A = prod u_i[idx_i], B = prod v_i[idx_i]  =>
    # C[x] = alpha * prod_{extA} u * prod_{extB} v * prod_{int} (sum_t u_j[t] v_j[t])
    c, a, b = tcinputs.split_expr(expr)
    u = tcinputs.outer_factors(a, ext, 11)
    v = tcinputs.outer_factors(b, ext, 12)
    A, B = tcinputs.outer_tensor(a, u), tcinputs.outer_tensor(b, v)
    alpha = 0.75
    got, S = oracle.contract(expr, _ext_str(ext, a + b), A, B, alpha=alpha, with_scale=True)
    fac = {x: (u[x] if x in a else v[x]) for x in c}
    want = alpha * tcinputs.outer_tensor(c, fac)
    for j in a:
        if j not in c:
            want = want * float(np.dot(u[j], v[j]))
    assert np.all(np.abs(got - want) <= TAU64 * S)


def test_constant_inputs():
    ext = {"a": 3, "b": 4, "c": 5, "d": 6, "e": 7, "f": 8}
    es = _ext_str(ext, "abcdef")
    got = oracle.contract("abcd-aebf-dfce", es, np.ones(3 * 7 * 4 * 8), np.ones(6 * 8 * 5 * 7),
                          alpha=2.0)
    assert np.all(got == 2.0 * 7 * 8)


def test_delta_inputs_give_permutation():
    # eq. (1) with N_e = N_c, N_f = N_d and B = delta(e,c) delta(f,d):
    # C[a,b,c,d] = A[a,c,b,d] (a pure permutation of A), bitwise.
    ext = {"a": 3, "b": 4, "c": 5, "d": 2, "e": 5, "f": 2}
    A = tcinputs.uniform_np(3 * 5 * 4 * 2, 5)
    Bn = np.zeros((5, 5, 2, 2))                 # axes e, c, f, d  (B[d,f,c,e])
    for i in range(5):
        for j in range(2):
            Bn[i, i, j, j] = 1.0
    got = oracle.contract("abcd-aebf-dfce", _ext_str(ext, "abcdef"), A, Bn.reshape(-1))
    An = A.reshape(2, 4, 5, 3)                  # axes f(=d), b, e(=c), a
    want = np.transpose(An, (0, 2, 1, 3)).reshape(-1)   # axes d, c, b, a
    assert np.array_equal(got, want)


def test_linearity_alpha_beta_and_nan():
    ext = {"a": 4, "b": 5, "c": 3, "d": 6, "e": 7}
    es, expr = _ext_str(ext, "abcde"), "abcd-dbea-ec"
    nA, nB, nC = 6 * 5 * 7 * 4, 7 * 3, 4 * 5 * 3 * 6
    A1, A2 = tcinputs.uniform_np(nA, 1), tcinputs.uniform_np(nA, 2)
    B = tcinputs.uniform_np(nB, 3)
    C0 = tcinputs.uniform_np(nC, 4)
    lam, mu = 0.3, -1.7
    lhs, S = oracle.contract(expr, es, lam * A1 + mu * A2, B, with_scale=True)
    r1, S1 = oracle.contract(expr, es, A1, B, with_scale=True)
    r2, S2 = oracle.contract(expr, es, A2, B, with_scale=True)
    assert np.all(np.abs(lhs - (lam * r1 + mu * r2)) <= 4 * TAU64 * (abs(lam) * S1 + abs(mu) * S2))
    got = oracle.contract(expr, es, A1, B, C=C0, alpha=0.5, beta=-2.0)
    assert np.all(np.abs(got - (0.5 * r1 - 2.0 * C0)) <= TAU64 * (0.5 * S1 + 2 * np.abs(C0)))
    nanC = np.full(nC, np.nan)
    got = oracle.contract(expr, es, A1, B, C=nanC, alpha=1.0, beta=0.0)
    assert np.all(np.isfinite(got)) and np.array_equal(got, r1)


def test_relabelling_invariance():
    ext = {"a": 3, "b": 2, "c": 4, "d": 5, "e": 3, "f": 2}
    A = tcinputs.uniform_np(3 * 3 * 2 * 2, 8)
    B = tcinputs.uniform_np(5 * 2 * 4 * 3, 9)
    r1 = oracle.contract("abcd-aebf-dfce", _ext_str(ext, "abcdef"), A, B)
    ren = dict(zip("abcdef", "qzxwvu"))
    ext2 = {ren[k]: v for k, v in ext.items()}
    expr2 = "".join(ren.get(ch, ch) for ch in "abcd-aebf-dfce")
    r2 = oracle.contract(expr2, _ext_str(ext2, "".join(ext2)), A, B)
    assert np.array_equal(r1, r2)


def test_operand_swap_and_output_permutation():
    ext = {"a": 3, "b": 2, "c": 4, "d": 5, "e": 3, "f": 2}
    es = _ext_str(ext, "abcdef")
    A = tcinputs.integers_np(3 * 3 * 2 * 2, 8)
    B = tcinputs.integers_np(5 * 2 * 4 * 3, 9)
    r1 = oracle.contract("abcd-aebf-dfce", es, A, B)
    assert np.array_equal(r1, oracle.contract("abcd-dfce-aebf", es, B, A))
    r3 = oracle.contract("dcba-aebf-dfce", es, A, B)       # C'[d,c,b,a] = C[a,b,c,d]
    Cn = r1.reshape(5, 4, 2, 3)                              # axes d, c, b, a
    assert np.array_equal(r3, np.transpose(Cn, (3, 2, 1, 0)).reshape(-1))


def test_slab_and_sample_consistency():
    ext = {"a": 5, "b": 4, "c": 3, "d": 5, "e": 4, "f": 3, "g": 6}
    es, expr = _ext_str(ext, "abcdefg"), "abcdef-gdab-efgc"
    A = tcinputs.uniform_np(6 * 5 * 5 * 4, 1)
    B = tcinputs.uniform_np(4 * 3 * 6 * 3, 2)
    full = oracle.contract(expr, es, A, B)
    cuts = [0, 7, 500, 501, 1999, full.size]
    parts = [oracle.contract(expr, es, A, B, lo=lo, hi=hi) for lo, hi in zip(cuts[:-1], cuts[1:])]
    assert np.array_equal(np.concatenate(parts), full)
    idx = np.array([0, 17, full.size - 1, 1234, 17])
    assert np.array_equal(oracle.sample(expr, es, A, B, idx), full[idx])
    # slab of C's slowest index f: [lo, hi) of f is a contiguous C range
    per_f = full.size // 3
    slab = oracle.contract(expr, es, A, B, lo=per_f, hi=2 * per_f)
    assert np.array_equal(slab, full[per_f:2 * per_f])


def test_neumaier_against_fsum():
    ext = {"a": 3, "b": 2, "c": 5184}
    es = _ext_str(ext, "abc")
    A = tcinputs.uniform_np(3 * 5184, 21)
    B = tcinputs.uniform_np(5184 * 2, 22)
    ex = oracle.contract("ab-ac-cb", es, A, B, exact=True)
    pl, S = oracle.contract("ab-ac-cb", es, A, B, with_scale=True)
    MA, MB = A.reshape(5184, 3).T, B.reshape(2, 5184).T
    for i in range(3):
        for j in range(2):
            f = math.fsum(MA[i, k] * MB[k, j] for k in range(5184))
            # the products themselves are rounded; fsum sums the same rounded products
            assert abs(ex[i + 3 * j] - f) <= 2.3e-16 * abs(f) + 1e-300
            assert abs(pl[i + 3 * j] - f) <= 5184 * 1.2e-16 * S[i + 3 * j]


def _bf16_round_check(terms):
    """Contract bf16 terms with ones (exact fp64 sum s) and check RNE of s to bf16."""
    a = tcinputs.bf16_bits(terms)
    assert np.array_equal(tcinputs.bf16_to_f64(a), np.asarray(terms, dtype=np.float64))
    n = len(terms)
    s = math.fsum(terms)
    r = oracle.contract("a-ac-c", f"a:1;c:{n}", a, tcinputs.bf16_bits([1.0] * n), dtype="bf16")[0]
    rv = tcinputs.bf16_to_f64([r])[0]
    up = tcinputs.bf16_to_f64([np.uint16(r + 1)])[0]
    dn = tcinputs.bf16_to_f64([np.uint16(r - 1)])[0] if r & 0x7FFF else -rv
    # rv is a nearest bf16 neighbour of s; on a tie the mantissa is even
    assert abs(rv - s) <= abs(up - s) and abs(rv - s) <= abs(dn - s), (terms, s, rv)
    if abs(rv - s) in (abs(up - s), abs(dn - s)) and rv != s:
        assert r % 2 == 0
    return rv


def test_bf16_output_rounding_is_rne():
    rng = np.random.default_rng(0)
    for _ in range(300):
        t = tcinputs.bf16_to_f64(tcinputs.bf16_bits(rng.uniform(-2, 2, 3) * 2.0 ** rng.integers(-12, 3, 3)))
        _bf16_round_check(list(t))
    # double-rounding trap: 1 + 2^-8 + 2^-40 rounds UP to 1 + 2^-7 (via f32 it would tie to 1)
    assert _bf16_round_check([1.0, 2.0 ** -8, 2.0 ** -40]) == 1.0 + 2.0 ** -7
    # exact tie rounds to even
    assert _bf16_round_check([1.0, 2.0 ** -8]) == 1.0
    assert _bf16_round_check([1.0 + 2.0 ** -7, 2.0 ** -8]) == 1.0 + 2.0 ** -6


def test_f32_path_rounds_once():
    # f32 inputs upcast exactly; output = (float) of the fp64 result (RNE)
    A = np.array([1.0, 2 ** -30], dtype=np.float32)
    B = np.array([1.0, 1.0], dtype=np.float32)
    r = oracle.contract("a-ac-c", "a:1;c:2", A, B, dtype="f32")
    assert r[0] == np.float32(1.0 + 2 ** -30)


# Batch (Hadamard) indices (R31): an index in C, A and B is
# not summed.  Pinned against torch.einsum and against per-slice TTGT (explicit slicing).
BATCH_CASES = [
    ("hij-hik-hkj", {"h": 3, "i": 4, "j": 5, "k": 6}),        # batched GEMM, batch fastest
    ("ijh-ikh-kjh", {"h": 3, "i": 4, "j": 5, "k": 2}),        # batch slowest
    ("abcd-aebd-ecd", {"a": 2, "b": 3, "c": 4, "d": 3, "e": 5}),
    ("ab-ab-ab", {"a": 5, "b": 7}),                            # pure Hadamard product
    ("abc-ab-cb", {"a": 3, "b": 4, "c": 5}),                   # batched outer product
    ("C[h,g,i] = A[g,k,h] * B[k,i,g,h]", {"h": 2, "g": 3, "i": 4, "k": 5}),
]


@pytest.mark.parametrize("expr,ext", BATCH_CASES)
def test_batch_indices_vs_einsum_and_sliced_ttgt(expr, ext):
    import re
    if "[" in expr:
        c, a, b = ("".join(re.findall(r"[a-z]", t)) for t in
                   re.match(r"C\[(.*)\] = A\[(.*)\] \* B\[(.*)\]", expr).groups())
    else:
        c, a, b = tcinputs.split_expr(expr)
    es = _ext_str(ext, a + b)
    A = tcinputs.uniform_np(tcinputs.numel(a, ext), 31)
    B = tcinputs.uniform_np(tcinputs.numel(b, ext), 32)
    got, S = oracle.contract(expr, es, A, B, with_scale=True)
    assert np.all(np.abs(got - einsum_ref(c, a, b, ext, A, B)) <= TAU64 * S)
    Ai, Bi = tcinputs.integers_np(A.size, 33), tcinputs.integers_np(B.size, 34)
    from tests.ttgt import batched_ttgt
    assert np.array_equal(oracle.contract(expr, es, Ai, Bi), batched_ttgt(c, a, b, ext, Ai, Bi))


# ---------------------------------------------------------------------------------------
# The tolerance scale S[x] = |alpha| sum_y |A B| + |beta| |C_in[x]| (SURVEY 8(c) "Tolerance",
# DESIGN R29) decides every random-data parity test, so it is pinned on its own: against
# torch.einsum of |A| and |B| (an independent formulation), and against the closed form
# S = |C| for all-positive inputs.  An over-estimated S (e.g. x K) would loosen every test.
@pytest.mark.parametrize("case", [c for c in tcinputs.tccg48()], ids=lambda c: f"tccg{c.id}")
def test_tolerance_scale_s_vs_einsum_of_abs(case):
    c, a, b = tcinputs.split_expr(case.expr)
    primes = [2, 3, 5, 2, 3, 4, 3, 2]
    ext = {x: primes[i % len(primes)] for i, x in enumerate(sorted(set(a + b)))}
    es = _ext_str(ext, a + b)
    A = tcinputs.uniform_np(tcinputs.numel(a, ext), 1100 + case.id)
    B = tcinputs.uniform_np(tcinputs.numel(b, ext), 2100 + case.id)
    C0 = tcinputs.uniform_np(tcinputs.numel(c, ext), 3100 + case.id)
    alpha, beta = -0.7, 1.3
    _, S = oracle.contract(case.expr, es, A, B, C=C0, alpha=alpha, beta=beta, with_scale=True)
    want = abs(alpha) * einsum_ref(c, a, b, ext, np.abs(A), np.abs(B)) + abs(beta) * np.abs(C0)
    assert np.allclose(S, want, rtol=1e-13, atol=0)
    # beta = 0: no C term (the old C is not read, R3)
    _, S0 = oracle.contract(case.expr, es, A, B, alpha=alpha, with_scale=True)
    assert np.allclose(S0, abs(alpha) * einsum_ref(c, a, b, ext, np.abs(A), np.abs(B)), rtol=1e-13, atol=0)
    # sample mode gives the same S as range mode, element by element
    idx = np.arange(0, S.size, 3)
    _, Ss = oracle.sample(case.expr, es, A, B, idx, C=C0, alpha=alpha, beta=beta, with_scale=True)
    assert np.array_equal(Ss, S[idx])


def test_tolerance_scale_equals_result_for_positive_inputs():
    # all terms positive => sum |A B| = sum A B exactly in the same order: S == C bitwise
    expr, ext = "abcd-aebf-dfce", {"a": 3, "b": 4, "c": 5, "d": 2, "e": 7, "f": 3}
    es = _ext_str(ext, "abcdef")
    A = np.abs(tcinputs.uniform_np(3 * 7 * 4 * 3, 5)) + 0.1
    B = np.abs(tcinputs.uniform_np(2 * 3 * 5 * 7, 6)) + 0.1
    got, S = oracle.contract(expr, es, A, B, with_scale=True)
    assert np.array_equal(got, S)
    got, S = oracle.contract(expr, es, A, B, alpha=2.0, with_scale=True)
    assert np.array_equal(got, S)
