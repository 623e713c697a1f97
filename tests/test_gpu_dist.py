"""GPU checks of the multi-GPU building blocks (dist.py) on one B200 — the data
path of the sharded modes through libtc's kernels, NCCL at world size 1:
  * C-slab sharding with the scattered input: the rank's sub-plan reads a compact slab of A
    (TC_SLAB_A) and writes a compact slab of C (TC_SLAB_C);
  * split-K with FP32 partials of a BF16 contraction (plan option out_f32): two k-halves as
    FP32 partials, summed, rounded once by tc_round_bf16 — bit-exact against the oracle's
    single rounding of the exact sum (integer data, |partial| < 2^24);
  * execute_split_k end to end over NCCL (reduce-scatter at world size 1).
Needs a B200: run with -m gpu."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build, dist as tcdist

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)
    if not dist.is_initialized():
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(_free_port()))
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    yield
    if dist.is_initialized():
        dist.destroy_process_group()


def _bf16(x):
    return torch.from_numpy(tcinputs.bf16_bits(x).view(np.int16).copy()).view(torch.bfloat16).cuda()


def _bits(t):
    return t.cpu().view(torch.int16).numpy().view(np.uint16)


def test_scatter_slab_world1():
    expr, extents = "abc-adc-db", "a:40;b:36;c:90;d:30"
    plan = tc.plan(expr, extents)
    sh = tcdist.shard_plan(plan, expr, extents, 1, 0)
    assert sh.x_tensor == "A" and sh.x_slabs == [(0, 40 * 30 * 90)]
    A = torch.from_numpy(tcinputs.integers_np(plan.numel("A"), 3)).cuda()
    B = torch.from_numpy(tcinputs.integers_np(plan.numel("B"), 4)).cuda()
    C = torch.full((sh.c_numel,), float("nan"), dtype=torch.float64, device="cuda")
    tcdist.execute_sharded(sh, A, B, C, rank=0)
    torch.cuda.synchronize()
    want = oracle.contract(expr, extents, A.cpu().numpy(), B.cpu().numpy())
    assert np.array_equal(C.cpu().numpy(), want)


def test_split_k_fp32_partials_bf16():
    expr, extents = "ab-ac-cb", "a:256;b:192;c:6000"
    Ah = tcinputs.integers_np(256 * 6000, 5)
    Bh = tcinputs.integers_np(6000 * 192, 6)
    A, B = _bf16(Ah), _bf16(Bh)
    base = tc.plan(expr, extents, dtype="bf16", out_f32=True)
    assert base.info()["out_f32"] == 1
    parts = []
    for lo, ln in ((0, 3100), (3100, 2900)):
        sub = base.restrict("c", lo, ln)
        Cp = torch.full((256 * 192,), float("nan"), dtype=torch.float32, device="cuda")
        sub.execute(A, B, Cp)
        parts.append(Cp)
    tot = parts[0] + parts[1]                       # (the reduce-scatter's sum, in the test)
    out = torch.empty(256 * 192, dtype=torch.bfloat16, device="cuda")
    tc.round_bf16(out, tot)
    torch.cuda.synchronize()
    want = oracle.contract(expr, extents, tcinputs.bf16_bits(Ah), tcinputs.bf16_bits(Bh), dtype="bf16")
    assert np.array_equal(_bits(out), want)
    # end to end through execute_split_k over NCCL (world size 1)
    sub, k, lo, ln = tcdist.split_k_plan(base, expr, extents, 1, 0)
    n = 256 * 192
    Cp = torch.zeros(tcdist.partial_numel(n, 1), dtype=torch.float32, device="cuda")
    res = torch.empty(n, dtype=torch.bfloat16, device="cuda")
    got = tcdist.execute_split_k(sub, A, B, Cp, 1, 0, n=n, out_bf16=res)
    torch.cuda.synchronize()
    assert np.array_equal(_bits(got), want)
