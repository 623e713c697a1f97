"""GPU parity of tc_execute_group (first step): the 18 CCSD(T)
sd_t_d1 / sd_t_d2 contractions of TCCG-48 (cases 31-48) accumulated into one t3,
C = alpha * sum_i contraction_i + beta * C, against the sum of the oracle's contractions on the
same seeded inputs.  Extents are ragged primes-ish so every tile has a tail.  Needs a B200."""
import numpy as np
import pytest
import torch

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build

pytestmark = pytest.mark.gpu
TAU64 = 1e-12
EXT = "a:6;b:5;c:7;d:6;e:5;f:7;g:9"


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


def _triples():
    return [c.expr for c in tcinputs.tccg48() if c.group.startswith("CCSDT")]


def _inputs(exprs, gen, plans):
    A = [gen(p.numel("A"), 100 + i) for i, p in enumerate(plans)]
    B = [gen(p.numel("B"), 200 + i) for i, p in enumerate(plans)]
    return A, B


def _oracle_sum(exprs, A, B, C0, alpha, beta):
    want = beta * C0 if C0 is not None else 0.0
    S = abs(beta) * np.abs(C0) if C0 is not None else 0.0
    for e, a, b in zip(exprs, A, B):
        w, s = oracle.contract(e, EXT, a, b, alpha=alpha, with_scale=True)
        want = want + w
        S = S + s
    return want, S


@pytest.mark.parametrize("integer", [True, False])
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (0.5, -2.0)])
def test_ccsdt_triples_group(integer, alpha, beta):
    exprs = _triples()
    assert len(exprs) == 18
    plans = [tc.plan(e, EXT) for e in exprs]
    gen = tcinputs.integers_np if integer else tcinputs.uniform_np
    A, B = _inputs(exprs, gen, plans)
    n = plans[0].numel("C")
    C0 = gen(n, 300) if beta != 0 else None
    dA = [torch.as_tensor(np.ascontiguousarray(a), device="cuda") for a in A]
    dB = [torch.as_tensor(np.ascontiguousarray(b), device="cuda") for b in B]
    dC = (torch.as_tensor(C0, device="cuda").clone() if C0 is not None
          else torch.full((n,), float("nan"), dtype=torch.float64, device="cuda"))
    tc.execute_group(plans, dA, dB, dC, alpha, beta)
    torch.cuda.synchronize()
    got = dC.cpu().numpy()
    want, S = _oracle_sum(exprs, A, B, C0, alpha, beta)
    if integer:
        assert np.array_equal(got, want), np.flatnonzero(got != want)[:10]
    else:
        bad = np.flatnonzero(~(np.abs(got - want) <= TAU64 * S))
        assert bad.size == 0, (bad[:10], got[bad[:3]], want[bad[:3]])


def test_group_in_cuda_graph():
    """The group is capturable: one graph replays the 18 launches (and gives the same C)."""
    exprs = _triples()
    plans = [tc.plan(e, EXT) for e in exprs]
    A, B = _inputs(exprs, tcinputs.integers_np, plans)
    dA = [torch.as_tensor(np.ascontiguousarray(a), device="cuda") for a in A]
    dB = [torch.as_tensor(np.ascontiguousarray(b), device="cuda") for b in B]
    n = plans[0].numel("C")
    dC = torch.zeros(n, dtype=torch.float64, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        tc.execute_group(plans, dA, dB, dC)        # warm-up outside capture
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        tc.execute_group(plans, dA, dB, dC)
    dC.fill_(float("nan"))
    g.replay()
    torch.cuda.synchronize()
    want, _ = _oracle_sum(exprs, A, B, None, 1.0, 0.0)
    assert np.array_equal(dC.cpu().numpy(), want)


def test_group_with_members_tuned_at_beta1():
    """tc_plan_tuned_beta: accumulating members tuned at beta = 1 still compute the group."""
    exprs = _triples()
    plans = [tc.plan(e, EXT) for e in exprs]
    A, B = _inputs(exprs, tcinputs.integers_np, plans)
    dA = [torch.as_tensor(np.ascontiguousarray(a), device="cuda") for a in A]
    dB = [torch.as_tensor(np.ascontiguousarray(b), device="cuda") for b in B]
    n = plans[0].numel("C")
    dC = torch.zeros(n, dtype=torch.float64, device="cuda")
    plans = [p.tuned(dA[i], dB[i], dC, topk=3, reps=1, beta=0.0 if i == 0 else 1.0)
             for i, p in enumerate(plans)]
    assert all(len(p.info()["stats"]["tuned"]) >= 1 for p in plans)
    dC.fill_(float("nan"))
    tc.execute_group(plans, dA, dB, dC)
    torch.cuda.synchronize()
    want, _ = _oracle_sum(exprs, A, B, None, 1.0, 0.0)
    assert np.array_equal(dC.cpu().numpy(), want)
