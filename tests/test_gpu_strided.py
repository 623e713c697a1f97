"""GPU parity of plans over caller-given strides (tc_plan_strided; SURVEY 8(a) row f3 /
NEXT-3) against the CPU oracle.  The strided buffers are gathered into the dense
layout on the host (numpy views, no arithmetic), the oracle contracts the dense tensors, and
the expected C is scattered back into a copy of the initial C buffer: every element outside
the view must come back unchanged (no stray writes), every element inside bit-exact on
integer data (FP64 and BF16).  Needs a B200: run with -m gpu."""
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


def _view(buf, idx, ext, strides):
    """numpy view of a strided tensor in the dense convention (first letter fastest)."""
    shape = tuple(ext[x] for x in reversed(idx))
    st = tuple(buf.itemsize * s for s in reversed(strides))
    return np.lib.stride_tricks.as_strided(buf, shape=shape, strides=st)


def _dense_strides(idx, ext):
    s, out = 1, []
    for x in idx:
        out.append(s)
        s *= ext[x]
    return out


# (expr, extents, strides per tensor; None = dense)
CASES = [
    # padded leading dimensions (pitch) on every tensor
    ("ab-ac-cb", "a:70;b:50;c:40", {"C": [1, 72], "A": [1, 80], "B": [1, 48]}),
    # A stored transposed relative to the expression's letter order, C with gaps
    ("ab-ac-cb", "a:64;b:33;c:40", {"C": [2, 160], "A": [40, 1]}),
    # 4D with a broadcast (stride 0) input index and permuted strides
    ("abcd-aebf-dfce", "a:12;b:10;c:9;d:8;e:7;f:6",
     {"A": [1, 12 * 10 * 7, 12, 12 * 7], "B": [1, 8, 8 * 6 * 9, 8 * 6], "C": [1, 13, 13 * 11, 13 * 11 * 10]}),
    ("abc-abd-dc", "a:16;b:9;c:12;d:20", {"A": [0, 1, 9], "C": [1, 17, 17 * 10]}),
    # the TCCG #1 layout with a padded FVI pitch on A and C
    ("abcde-efbad-cf", "a:10;b:6;c:8;d:5;e:12;f:9",
     {"A": [1, 16, 16 * 9, 16 * 9 * 6, 16 * 9 * 6 * 10], "C": [1, 16, 16 * 6, 16 * 6 * 8, 16 * 6 * 8 * 5]}),
]


def _run(expr, ext_s, strides, dtype, seed, beta=0.0):
    ext = tcinputs.parse_extents(ext_s)
    cidx, aidx, bidx = tcinputs.split_expr(expr)
    p = tc.plan_strided(expr, ext_s, strides, dtype=dtype)
    full = {t: (strides.get(t) or _dense_strides(i, ext)) for t, i in (("C", cidx), ("A", aidx), ("B", bidx))}
    idx = {"C": cidx, "A": aidx, "B": bidx}
    # storage arrays: float64, or BF16 bit patterns (uint16) — integers in [-3, 3] either way
    vals = {t: tcinputs.integers_np(p.span(t), 100 * seed + k) for k, t in enumerate("CAB")}
    bufs = {t: (vals[t].astype(np.float64) if dtype == "f64" else tcinputs.bf16_bits(vals[t])) for t in "CAB"}
    dense = {t: np.ascontiguousarray(_view(bufs[t], idx[t], ext, full[t])).reshape(-1) for t in "CAB"}
    want = oracle.contract(expr, ext_s, dense["A"], dense["B"], C=dense["C"] if beta else None, beta=beta,
                           dtype=dtype)
    expect = bufs["C"].copy()
    _view(expect, cidx, ext, full["C"])[...] = want.reshape(tuple(ext[x] for x in reversed(cidx)))
    if dtype == "f64":
        dev = {t: torch.from_numpy(bufs[t]).cuda() for t in "CAB"}
    else:
        dev = {t: torch.from_numpy(bufs[t].view(np.int16).copy()).view(torch.bfloat16).cuda() for t in "CAB"}
    p.execute(dev["A"], dev["B"], dev["C"], beta=beta)
    torch.cuda.synchronize()
    got = dev["C"].cpu()
    got = got.numpy() if dtype == "f64" else got.view(torch.int16).numpy().view(np.uint16)
    bad = np.flatnonzero(got != expect)
    assert bad.size == 0, (expr, dtype, bad[:10], got[bad[:3]], expect[bad[:3]])


@pytest.mark.parametrize("i", range(len(CASES)))
@pytest.mark.parametrize("dtype", ["f64", "bf16"])
def test_strided_parity(i, dtype):
    expr, ext, strides = CASES[i]
    _run(expr, ext, strides, dtype, seed=i)
    _run(expr, ext, strides, dtype, seed=i + 7, beta=1.0)
