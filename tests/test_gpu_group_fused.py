"""GPU parity of the FUSED grouped contraction (tc_group_plan / tc_group_execute; SURVEY 8(f)
NEXT-4, R34): one kernel computes C = alpha * sum_i contraction_i + beta * C with
every C tile kept on chip across the members and stored once.  Checked against the sum of
the oracle's contractions on the same seeded inputs (integer data: bitwise; random data:
|C - C_ref| <= tau * sum_i S_i), for the 18 CCSD(T) triples (TCCG #31-48) at
ragged extents (partial tiles on every C index), at the TCCG extents and uniform N (sampled),
with k padding (Kt < BK), several k-steps per member, misaligned pointers, and inside a CUDA
graph.  Needs a B200."""
import numpy as np
import pytest
import torch

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build

pytestmark = pytest.mark.gpu
TAU64 = 1e-12
RAGGED = "a:6;b:5;c:7;d:6;e:5;f:7;g:9"


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


def triples():
    return [c.expr for c in tcinputs.tccg48() if c.group.startswith("CCSDT")]


def oracle_sum(exprs, ext, A, B, C0, alpha, beta, idx=None):
    """sum_i oracle(contraction_i) (alpha applied per member, beta on the old C): the oracle's
    own results added, no new arithmetic (DESIGN R33); idx = sampled C linear indices."""
    want, S = 0.0, 0.0
    if C0 is not None:
        c0 = C0 if idx is None else C0[idx]
        want, S = beta * c0, abs(beta) * np.abs(c0)
    for e, a, b in zip(exprs, A, B):
        if idx is None:
            w, s = oracle.contract(e, ext, a, b, alpha=alpha, with_scale=True)
        else:
            w, s = oracle.sample(e, ext, a, b, idx, alpha=alpha, with_scale=True)
        want, S = want + w, S + s
    return want, S


def run_fused(exprs, ext, A, B, C0, alpha=1.0, beta=0.0, misalign=0):
    plans = [tc.plan(e, ext) for e in exprs]
    g = tc.plan_group(plans)
    n = plans[0].numel("C")

    def dev(x):
        t = torch.empty(x.size + misalign, dtype=torch.float64, device="cuda")
        t[misalign:] = torch.as_tensor(np.ascontiguousarray(x))
        return t[misalign:]
    dA, dB = [dev(a) for a in A], [dev(b) for b in B]
    if C0 is not None:
        dC = dev(C0)
    else:
        dC = torch.full((n + misalign,), float("nan"), dtype=torch.float64, device="cuda")[misalign:]
    g.execute(dA, dB, dC, alpha, beta)
    torch.cuda.synchronize()
    return g, dC


def inputs(exprs, ext, gen):
    plans = [tc.plan(e, ext, host_only=True) for e in exprs]
    A = [gen(p.numel("A"), 100 + i) for i, p in enumerate(plans)]
    B = [gen(p.numel("B"), 200 + i) for i, p in enumerate(plans)]
    return A, B, plans[0].numel("C")


@pytest.mark.parametrize("integer", [True, False])
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (0.5, -2.0), (-1.0, 1.0)])
def test_triples_fused_ragged(integer, alpha, beta):
    exprs = triples()
    gen = tcinputs.integers_np if integer else tcinputs.uniform_np
    A, B, n = inputs(exprs, RAGGED, gen)
    C0 = gen(n, 300) if beta != 0 else None
    g, dC = run_fused(exprs, RAGGED, A, B, C0, alpha, beta)
    i = g.info()
    assert i["members"] == 18 and any(n % t for n, t in zip((6, 5, 7, 6, 5, 7), i["T"]))  # partial tiles
    got = dC.cpu().numpy()
    want, S = oracle_sum(exprs, RAGGED, A, B, C0, alpha, beta)
    if integer:
        assert np.array_equal(got, want), np.flatnonzero(got != want)[:10]
    else:
        bad = np.flatnonzero(~(np.abs(got - want) <= TAU64 * S))
        assert bad.size == 0, (bad[:10], got[bad[:3]], want[bad[:3]])


@pytest.mark.parametrize("misalign", [1, 3])
def test_triples_fused_misaligned_pointers(misalign):
    # 8-B aligned only: scalar cp.async and scalar C stores (vector paths off at run time)
    exprs = triples()
    A, B, n = inputs(exprs, RAGGED, tcinputs.integers_np)
    C0 = tcinputs.integers_np(n, 301)
    g, dC = run_fused(exprs, RAGGED, A, B, C0, 1.0, 1.0, misalign=misalign)
    want, _ = oracle_sum(exprs, RAGGED, A, B, C0, 1.0, 1.0)
    assert np.array_equal(dC.cpu().numpy(), want)


@pytest.mark.parametrize("ext", ["a:24;b:16;c:16;d:24;e:16;f:16;g:24",          # TCCG #31-48
                                 ";".join(f"{x}:16" for x in "abcdefg"),          # bench N = 16 (BK 16)
                                 ";".join(f"{x}:24" for x in "abcdefg"),          # bench N = 24 (BK 24)
                                 "a:8;b:8;c:8;d:8;e:8;f:8;g:20"])                  # Kt = 20 < BK: k padding
def test_triples_fused_full_size_sampled(ext):
    exprs = triples()
    A, B, n = inputs(exprs, ext, tcinputs.integers_np)
    g, dC = run_fused(exprs, ext, A, B, None)
    rng = np.random.default_rng(7)
    idx = np.unique(np.concatenate([rng.integers(0, n, 1 << 14), np.arange(min(n, 4096)),
                                    np.arange(max(0, n - 4096), n)]))
    got = dC[torch.as_tensor(idx, device="cuda")].cpu().numpy()
    want, _ = oracle_sum(exprs, ext, A, B, None, 1.0, 0.0, idx=idx)
    assert np.array_equal(got, want), (g.info()["T"], idx[np.flatnonzero(got != want)[:10]])
    assert not bool(torch.isnan(dC).any())


def test_generic_group_several_ksteps_and_splits():
    # not triples: members with two internal indices (several k-steps at BK), different row /
    # column splits of C, and X = B for one member (C's FVI in B)
    exprs = ["abcd-aebf-dfce", "abcd-eafb-fdce", "abcd-ebfa-cdef", "abcd-cfed-ebaf"]
    ext = "a:9;b:10;c:11;d:6;e:7;f:13"
    for integer in (True, False):
        gen = tcinputs.integers_np if integer else tcinputs.uniform_np
        A, B, n = inputs(exprs, ext, gen)
        C0 = gen(n, 77)
        g, dC = run_fused(exprs, ext, A, B, C0, 0.75, 0.5)
        assert max(m["nsteps"] for m in g.info()["per_member"]) > 1
        got = dC.cpu().numpy()
        want, S = oracle_sum(exprs, ext, A, B, C0, 0.75, 0.5)
        if integer:
            assert np.array_equal(got, want)
        else:
            assert np.all(np.abs(got - want) <= TAU64 * S)


def test_fused_group_in_cuda_graph_and_repeatable():
    exprs = triples()
    A, B, n = inputs(exprs, RAGGED, tcinputs.integers_np)
    plans = [tc.plan(e, RAGGED) for e in exprs]
    g = tc.plan_group(plans)
    dA = [torch.as_tensor(a, device="cuda") for a in A]
    dB = [torch.as_tensor(b, device="cuda") for b in B]
    dC = torch.zeros(n, dtype=torch.float64, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        g.execute(dA, dB, dC)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph, stream=s):
        g.execute(dA, dB, dC)
    dC.fill_(float("nan"))
    graph.replay()
    torch.cuda.synchronize()
    want, _ = oracle_sum(exprs, RAGGED, A, B, None, 1.0, 0.0)
    assert np.array_equal(dC.cpu().numpy(), want)


def test_fused_equals_unfused_group():
    # the fused kernel and tc_execute_group (18 launches) compute the same sum (integer data)
    exprs = triples()
    ext = "a:8;b:12;c:8;d:12;e:8;f:4;g:16"
    A, B, n = inputs(exprs, ext, tcinputs.integers_np)
    plans = [tc.plan(e, ext) for e in exprs]
    dA = [torch.as_tensor(a, device="cuda") for a in A]
    dB = [torch.as_tensor(b, device="cuda") for b in B]
    c1 = torch.full((n,), float("nan"), dtype=torch.float64, device="cuda")
    c2 = torch.full((n,), float("nan"), dtype=torch.float64, device="cuda")
    tc.execute_group(plans, dA, dB, c1)
    tc.plan_group(plans).execute(dA, dB, c2)
    torch.cuda.synchronize()
    assert torch.equal(c1, c2)


def test_fused_group_errors():
    exprs = triples()
    plans = [tc.plan(e, RAGGED) for e in exprs]
    g = tc.plan_group(plans)
    d = torch.zeros(1 << 16, dtype=torch.float64, device="cuda")
    with pytest.raises(tc.TcError) as e:                    # C overlaps an input
        g.execute_ptr([d.data_ptr()] * 18, [d.data_ptr()] * 18, d.data_ptr())
    assert e.value.status == "TC_ERR_INVALID_ARG"
    with pytest.raises(tc.TcError) as e:                    # FP32 members
        tc.plan_group([tc.plan(exprs[0], RAGGED, dtype="f32")])
    assert e.value.status == "TC_ERR_UNSUPPORTED"
