"""GPU parity of the streaming path (stream.hpp / kernel_stream.cuh: Y whole in shared memory,
X by TMA boxes in its own order, C runs along its FVI from the MMA accumulators) through the C
ABI against the CPU oracle, in BF16 (the checks of test_gpu_bf16.check_bf16: integer data
bitwise, random data within one BF16 ulp + the FP32 accumulation bound), FP64 (1e-12 * S), TF32
and FP32-split (test_gpu_f32.check_f32).  Covers the three row modes (X's FVI external: SM_T;
X's FVI internal: SM_K; X's FVI = C's FVI: SM_M, FP64), edge tiles on every m dim, n not a
multiple of 8 and up to 72 on FP64, k not a multiple of 16, padding rows (odd octet counts),
alpha, beta on the path (FP64 / FP32 C), the model's alternative configurations, restricted
sub-plans, and the fall-backs to the plan's tile configuration (BF16 beta != 0, misaligned C).
Needs a B200: run with -m gpu."""
import numpy as np
import pytest
import torch

import oracle

import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build
from tests.test_gpu_bf16 import check_bf16
from tests.test_gpu_f32 import check_f32
from tests.test_gpu_parity import check_case

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


def _on(expr, ext):
    s = tc.plan(expr, ext, "bf16", host_only=True).info()["stream"]
    assert s["on"] == 1, s
    return s


# TCCG #1-8 shapes at reduced extents (first dims multiples of 8: 16-B TMA strides), both modes
REDUCED = [
    ("abcde-efbad-cf", "a:16;b:6;c:24;d:5;e:16;f:12"),     # SM_T (X's FVI e), #1
    ("abcde-efcad-bf", "a:24;b:20;c:5;d:3;e:24;f:12"),     # #2, n = 20
    ("abcd-dbea-ec", "a:24;b:9;c:24;d:24;e:24"),           # #3
    ("abcde-ecbfa-fd", "a:16;b:3;c:7;d:24;e:16;f:12"),     # #4
    ("abcd-deca-be", "a:24;b:24;c:5;d:16;e:24"),           # #5
    ("abc-bda-dc", "a:40;b:40;c:24;d:40"),                 # #6, 5 octets of b: a padding row set
    ("abcd-ebad-ce", "a:24;b:10;c:24;d:3;e:24"),           # SM_K (X's FVI e = k), #7
    ("abc-dca-bd", "a:40;b:24;c:21;d:40"),                 # SM_K, #8, rest product 21
]


@pytest.mark.parametrize("expr,ext", REDUCED, ids=[f"tccg{i + 1}" for i in range(8)])
def test_stream_tccg_shapes(expr, ext):
    _on(expr, ext)
    check_bf16(expr, ext, seed=1, integer=True, stream=True)
    check_bf16(expr, ext, seed=2, stream=True)
    check_bf16(expr, ext, seed=3, integer=True, alpha=-2.0, stream=True)


# edge tiles on every m dim, k padded to 16, n below a multiple of 8
RAGGED = [
    ("abcde-efbad-cf", "a:24;b:5;c:13;d:3;e:40;f:9"),
    ("abc-bda-dc", "a:56;b:24;c:7;d:300"),          # K = 300: several k-steps, the last partial
    ("abc-dca-bd", "a:40;b:17;c:21;d:40"),          # SM_K, rest rows 21 of 16-row sets: padding rows
    ("abcd-ebad-ce", "a:24;b:5;c:31;d:3;e:24"),     # SM_K, n = 31
    ("abcd-dbea-ec", "a:8;b:3;c:3;d:8;e:8"),        # one tile, n = 3
]


@pytest.mark.parametrize("expr,ext", RAGGED, ids=[f"r{i}" for i in range(len(RAGGED))])
def test_stream_ragged(expr, ext):
    p = tc.plan(expr, ext, "bf16", host_only=True)
    s = p.info()["stream"]
    if s["on"] != 1:
        pytest.skip(f"not a streaming shape: {s['why']}")
    check_bf16(expr, ext, seed=4, integer=True, stream=True)
    check_bf16(expr, ext, seed=5, stream=True)


def test_stream_fallbacks_beta_and_alignment():
    # beta != 0 and a C pointer off the run alignment take the plan's tcgen05 configuration:
    # same results
    expr, ext = REDUCED[0]
    _on(expr, ext)
    check_bf16(expr, ext, seed=6, integer=True, alpha=2.0, beta=1.0, stream=True)
    check_bf16(expr, ext, seed=7, integer=True, cmisalign=1, stream=True)
    check_bf16(expr, ext, seed=8, integer=True, misalign=8, stream=True)


def test_stream_off_matches():
    # the option turns the path off (tcgen05 configuration); both give the same bits on integers
    expr, ext = REDUCED[6]
    p = check_bf16(expr, ext, seed=9, integer=True, stream=False)
    assert p.info()["stream"]["on"] == 0


def test_stream_tuned_candidate():
    # tc_plan_tuned times the streaming path as candidate 99 beside the variants
    case = [c for c in tcinputs.tccg48() if c.id == 3][0]
    p = tc.plan(case.expr, case.extents, "bf16")
    assert p.info()["stream"]["on"] == 1
    A = tcinputs.uniform(p.numel("A"), 1, device="cuda").to(torch.bfloat16)
    B = tcinputs.uniform(p.numel("B"), 2, device="cuda").to(torch.bfloat16)
    C = torch.empty(p.numel("C"), dtype=torch.bfloat16, device="cuda")
    t = p.tuned(A, B, C, topk=2, reps=1)
    tried = [v for v, _ in t.info()["stats"]["tuned"]]
    assert 99 in tried and 98 in tried   # the streaming path's two best model configurations


def test_stream_ranks_agree():
    # the model's alternative streaming configurations (tc_plan_opts.stream_rank) give the same
    # bits on integer data
    for expr, ext in (REDUCED[0], REDUCED[6]):
        for r in (1, 2):
            p = tc.plan(expr, ext, "bf16", host_only=True, stream=True, stream_rank=r).info()["stream"]
            assert p["rank"] == min(r, p["nranks"] - 1)
            check_bf16(expr, ext, seed=30 + r, integer=True, stream=True, stream_rank=r)
            check_case(expr, ext, seed=40 + r, integer=True, stream=True, stream_rank=r, dtype="f64")


# FP64 (the paper's precision): DMMA m8n8k4 streaming kernel, tolerance 1e-12 * S (north_star)
@pytest.mark.parametrize("expr,ext", REDUCED + RAGGED, ids=[f"tccg{i + 1}" for i in range(8)] +
                         [f"r{i}" for i in range(len(RAGGED))])
def test_stream_f64(expr, ext):
    s = tc.plan(expr, ext, "f64", host_only=True, stream=True).info()["stream"]
    if s["on"] != 1:
        pytest.skip(f"not a streaming shape: {s['why']}")
    p = check_case(expr, ext, seed=11, integer=True, stream=True)
    assert p.info()["stream"]["active"] == 1
    check_case(expr, ext, seed=12, stream=True)
    check_case(expr, ext, seed=13, alpha=0.75, stream=True)
    check_case(expr, ext, seed=14, integer=True, alpha=2.0, beta=-1.0, stream=True)   # beta on the path
    check_case(expr, ext, seed=15, alpha=0.5, beta=1.5, stream=True)


# FP32 storage: TF32 products (R30 tolerance) and FP32 as split TF32 (1e-5 * S, R32)
@pytest.mark.parametrize("dtype", ["tf32", "f32"])
@pytest.mark.parametrize("expr,ext", REDUCED + RAGGED, ids=[f"tccg{i + 1}" for i in range(8)] +
                         [f"r{i}" for i in range(len(RAGGED))])
def test_stream_fp32(expr, ext, dtype):
    s = tc.plan(expr, ext, dtype, host_only=True, stream=True).info()["stream"]
    if s["on"] != 1:
        pytest.skip(f"not a streaming shape: {s['why']}")
    check_f32(expr, ext, dtype, seed=21, integer=True, stream=True)
    assert tc.plan(expr, ext, dtype, host_only=True, stream=True).info()["stream"]["active"] == 1
    check_f32(expr, ext, dtype, seed=22, stream=True)
    check_f32(expr, ext, dtype, seed=23, alpha=-1.5, stream=True)
    check_f32(expr, ext, dtype, seed=24, integer=True, alpha=2.0, beta=-1.0, stream=True)   # beta on the path
    check_f32(expr, ext, dtype, seed=25, alpha=0.5, beta=1.5, stream=True)


@pytest.mark.parametrize("expr,ext", [("abc-bda-dc", "a:24;b:40;c:40;d:24"),      # n = 40 (9 n8 blocks)
                                      ("abcd-ebad-ce", "a:16;b:8;c:72;d:2;e:24"),  # SM_K, n = 72
                                      ("abcde-efbad-cf", "a:16;b:3;c:57;d:2;e:16;f:12")])
def test_stream_f64_wide_n(expr, ext):
    # FP64 streaming with the Y-side extent up to 72 (NB = 9, AR = 2)
    s = tc.plan(expr, ext, "f64", host_only=True, stream=True).info()["stream"]
    assert s["on"] == 1 and s["NB"] == 9, s
    check_case(expr, ext, seed=51, integer=True, stream=True, dtype="f64")
    check_case(expr, ext, seed=52, stream=True, dtype="f64")


@pytest.mark.parametrize("expr,ext", [("abcd-eb-aecd", "a:16;b:24;c:8;d:4;e:16"),     # SM_M (X's FVI = C's FVI)
                                      ("abcd-eb-aecd", "a:24;b:19;c:5;d:3;e:13"),     # edges, k padded
                                      ("abcd-ec-abed", "a:16;b:3;c:72;d:8;e:24"),     # n = 72
                                      ("abcd-eb-aecd", "a:40;b:8;c:6;d:10;e:8")])    # 5 octets of a
def test_stream_f64_sm_m(expr, ext):
    # FP64 streaming with X's FVI = C's FVI: row octets along a, AR blocks over the next X dim
    s = tc.plan(expr, ext, "f64", host_only=True, stream=True, fusion=False).info()["stream"]
    assert s["on"] == 1 and s["mode"] == "M", s
    check_case(expr, ext, seed=61, integer=True, stream=True, dtype="f64", fusion=False)
    check_case(expr, ext, seed=62, stream=True, dtype="f64", fusion=False)
    check_case(expr, ext, seed=63, integer=True, alpha=-1.0, beta=2.0, stream=True, dtype="f64", fusion=False)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_stream_restricted_slabs(dtype):
    # the multi-GPU C-slab and split-K sub-plans (tc_plan_restrict) of a streaming
    # shape take the streaming path too (restricted views: bases, partial extents) — bitwise on
    # integers, slabs reassembling the full result
    expr, ext = "abcde-efbad-cf", "a:16;b:6;c:24;d:6;e:16;f:12"
    tdt = torch.float64 if dtype == "f64" else torch.float32
    p = tc.plan(expr, ext, dtype)
    assert p.info()["stream"]["active"] == 1
    A = tcinputs.integers_np(p.numel("A"), 71)
    B = tcinputs.integers_np(p.numel("B"), 72)
    full = oracle.contract(expr, ext, A, B)
    dA = torch.as_tensor(A, device="cuda").to(tdt)
    dB = torch.as_tensor(B, device="cuda").to(tdt)
    dC = torch.full((p.numel("C"),), float("nan"), dtype=tdt, device="cuda")
    for lo, ln in [(0, 2), (2, 3), (5, 1)]:        # C slabs on d (the slowest X external)
        sub = p.restrict("d", lo, ln)
        sub.execute(dA, dB, dC)
    torch.cuda.synchronize()
    assert np.array_equal(dC.double().cpu().numpy(), full)
    acc = torch.zeros_like(dC)
    for lo, ln in [(0, 5), (5, 7)]:                # split-K over f
        part = torch.zeros_like(dC)
        p.restrict("f", lo, ln).execute(dA, dB, part)
        acc += part
    torch.cuda.synchronize()
    assert np.array_equal(acc.double().cpu().numpy(), full)
