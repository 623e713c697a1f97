"""GPU parity of representative-size plans (tc_plan_resize / tc_plan_select; SURVEY 8(a) row
f1 / NEXT-1): a configuration chosen at one size runs correctly at others —
smaller, larger, ragged against its tiles — in FP64 and BF16, bit-exact on integer data
against the CPU oracle.  Needs a B200: run with -m gpu."""
import numpy as np
import pytest
import torch

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


def _check(p, expr, ext, dtype, seed):
    gen = tcinputs.integers_np
    A, B = gen(p.numel("A"), 10 + seed), gen(p.numel("B"), 20 + seed)
    if dtype == "f64":
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        dC = torch.full((p.numel("C"),), float("nan"), dtype=torch.float64, device="cuda")
        want = oracle.contract(expr, ext, A, B)
    else:
        Ab, Bb = tcinputs.bf16_bits(A), tcinputs.bf16_bits(B)
        dA = torch.from_numpy(Ab.view(np.int16).copy()).view(torch.bfloat16).cuda()
        dB = torch.from_numpy(Bb.view(np.int16).copy()).view(torch.bfloat16).cuda()
        dC = torch.full((p.numel("C"),), float("nan"), dtype=torch.bfloat16, device="cuda")
        want = oracle.contract(expr, ext, Ab, Bb, dtype="bf16")
    p.execute(dA, dB, dC)
    torch.cuda.synchronize()
    got = dC.cpu().numpy() if dtype == "f64" else dC.cpu().view(torch.int16).numpy().view(np.uint16)
    bad = np.flatnonzero(got != want)
    assert bad.size == 0, (expr, ext, dtype, bad[:8])


def _ext(expr, sizes):
    c, a, b = tcinputs.split_expr(expr)
    names = sorted(set(a + b))
    return ";".join(f"{x}:{sizes[i % len(sizes)]}" for i, x in enumerate(names))


@pytest.mark.parametrize("dtype", ["f64", "bf16"])
@pytest.mark.parametrize("expr", ["abcd-aebf-dfce", "ab-ac-cb", "abcdef-gdab-efgc", "abc-bda-dc"])
def test_resize_runs_at_other_sizes(expr, dtype):
    rep = tc.plan(expr, _ext(expr, [16]), dtype=dtype)
    for sizes in ([7, 5, 9, 3, 11, 6, 4], [24, 17, 20, 31, 19, 22, 18], [40, 33, 9, 12, 5, 27, 14]):
        ext = _ext(expr, sizes)
        p = rep.resize(ext)
        assert p.info()["resized"] == 1 and p.info()["variant"] == rep.info()["variant"]
        _check(p, expr, ext, dtype, seed=sum(sizes))


@pytest.mark.parametrize("dtype", ["f64", "bf16"])
def test_select_among_versions(dtype):
    expr = "abcd-aebf-dfce"
    versions = [tc.plan(expr, _ext(expr, [n]), dtype=dtype) for n in (8, 24, 48)]
    for sizes in ([10, 9, 11, 12, 7, 8], [30, 26, 28, 25, 27, 29]):
        ext = _ext(expr, sizes)
        p, chosen = tc.select(versions, ext)
        assert 0 <= chosen < 3 and p.info()["resized"] == 1
        _check(p, expr, ext, dtype, seed=chosen + sum(sizes))
