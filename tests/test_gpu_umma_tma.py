"""GPU parity of the tcgen05 kernel with TMA operand boxes (kernel_umma.cuh TMA producer,
tiles.cpp umma_tma_spec) against the CPU oracle, BF16 and TF32, on plans forced into every
box shape the spec admits: K-major / MN-major on either side, MN-major tiles of two atoms
(two boxes per stage), multi-digit boxes (rank 3-5, permuted map dims), k tiles below BK
(the MMAs skip the next step's k the K-major box brings along), a k tile equal to a ragged
extent (zero fill past the end), ragged tails everywhere, beta != 0, and misaligned
pointers (the call falls back to the cp.async instance).  Tolerances as in test_gpu_bf16.py /
test_gpu_f32.py; integer data is bit-exact.  Needs a B200: run with -m gpu."""
import pytest
import torch

from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build
from tests.test_gpu_bf16 import check_bf16
from tests.test_gpu_f32 import check_f32

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


# (expr, extents, forced tiles) per dtype family (BF16: E = BK = 64, TF32: E = BK = 32); the
# extents keep every operand stride a multiple of 16 B (a tensor-map requirement)
CASES = [
    # X MN-major (a, two 64-atoms) / Y K-major, ragged m, n and k
    ("ab-ac-cb", "a:200;b:150;c:136", "a:128;b:128;c:64", "a:200;b:150;c:136", "a:64;b:128;c:32"),
    # X K-major / Y MN-major
    ("ab-ca-bc", "a:256;b:136;c:192", "a:128;b:64;c:64", "a:256;b:136;c:192", "a:128;b:32;c:32"),
    # both MN-major, k tile below BK (a multiple of the MMA K)
    ("ab-ac-bc", "a:136;b:104;c:80", "a:64;b:128;c:48", "a:136;b:104;c:80", "a:32;b:64;c:16"),
    # both K-major
    ("ab-ca-cb", "a:128;b:64;c:72", "a:128;b:64;c:64", "a:128;b:64;c:72", "a:128;b:64;c:32"),
    # k tile = the whole ragged extent (not a multiple of the MMA K): zero fill past it
    ("ab-ac-cb", "a:152;b:70;c:24", "a:128;b:64;c:24", "a:152;b:70;c:20", "a:64;b:64;c:20"),
    # K-major X with a three-digit side box (rank-4 map), MN-major Y
    ("abcd-ebad-ce", "a:20;b:5;c:72;d:9;e:104", "a:16;b:2;d:4;c:64;e:64",
     "a:20;b:5;c:72;d:9;e:104", "a:16;b:2;d:4;c:32;e:32"),
    # MN-major X over two side digits (T0 = E, the second tiled), K-major Y
    ("abc-acd-db", "a:72;b:50;c:3;d:40", "a:64;c:2;b:64;d:32", "a:72;b:50;c:5;d:40", "a:32;c:4;b:64;d:32"),
    # rank-5 MN-major X (the TCCG #1 layout), ragged
    ("abcde-efbad-cf", "a:3;b:2;c:40;d:2;e:64;f:33", "a:1;b:2;c:40;d:1;e:64;f:32",
     "a:3;b:2;c:40;d:2;e:64;f:33", "a:1;b:2;c:40;d:2;e:32;f:32"),
]


def _plan_kw(tiles):
    return dict(force_tiles=tiles, morder="X")


@pytest.mark.parametrize("i", range(len(CASES)))
def test_bf16_tma_operands(i):
    expr, ext, tb, _, _ = CASES[i]
    hp = tc.plan(expr, ext, dtype="bf16", host_only=True, **_plan_kw(tb))
    assert hp.info()["tma_operands"] == 1, hp.info()
    check_bf16(expr, ext, seed=i, integer=True, **_plan_kw(tb))
    check_bf16(expr, ext, seed=i, integer=False, **_plan_kw(tb))
    check_bf16(expr, ext, seed=i + 50, integer=True, alpha=2.0, beta=1.0, **_plan_kw(tb))
    # misaligned operands: the map cannot be encoded, the cp.async instance runs
    check_bf16(expr, ext, seed=i, integer=True, misalign=1, **_plan_kw(tb))
    # the same plan without TMA operands agrees
    check_bf16(expr, ext, seed=i, integer=True, tma_operands=False, **_plan_kw(tb))


@pytest.mark.parametrize("i", range(len(CASES)))
def test_tf32_tma_operands(i):
    expr, _, _, ext, tt = CASES[i]
    hp = tc.plan(expr, ext, dtype="tf32", host_only=True, **_plan_kw(tt))
    assert hp.info()["tma_operands"] == 1, hp.info()
    check_f32(expr, ext, "tf32", seed=i, integer=True, **_plan_kw(tt))
    check_f32(expr, ext, "tf32", seed=i, integer=False, **_plan_kw(tt))
    check_f32(expr, ext, "tf32", seed=i + 50, integer=True, alpha=2.0, beta=1.0, **_plan_kw(tt))
    check_f32(expr, ext, "tf32", seed=i, integer=True, misalign=1, **_plan_kw(tt))


def test_planner_choice_uses_tma_on_ab_ac_cb():
    # the TCCG #18 GEMM at its BASELINE extents plans TMA-fed in both BF16 and TF32
    for dt in ("bf16", "tf32"):
        p = tc.plan("ab-ac-cb", "a:5136;b:5120;c:5136", dtype=dt, host_only=True)
        assert p.info()["tma_operands"] == 1, (dt, p.info())


def test_unaligned_box_origins_keep_cp_async():
    # tile origins along a box's first dim off a 16-B boundary (T = 68 BF16 / 100) cannot be
    # TMA boxes (the hardware faults on them): such plans keep the cp.async producers
    for tiles in ("a:128;b:68;c:64", "a:128;b:100;c:64"):
        hp = tc.plan("ab-ca-bc", "a:256;b:136;c:192", dtype="bf16", host_only=True, force_tiles=tiles)
        assert hp.info()["tma_operands"] == 0
        check_bf16("ab-ca-bc", "a:256;b:136;c:192", seed=3, integer=True, force_tiles=tiles)
    # K-major dim 0 = k: a k tile of 12 BF16 (24 B) steps off 16 B
    hp = tc.plan("ab-ca-cb", "a:128;b:64;c:72", dtype="bf16", host_only=True, force_tiles="a:128;b:64;c:12")
    assert hp.info()["tma_operands"] == 0
    check_bf16("ab-ca-cb", "a:128;b:64;c:72", seed=4, integer=True, force_tiles="a:128;b:64;c:12")


# CTA pairs (kernel_umma.cuh PAIR): clusters of two CTAs, M = 256 MMAs over 2 x 2 blocks of
# BN = 128 tiles; odd tile counts hand the overhanging block the padding entry
PAIR_CASES = [
    ("ab-ac-cb", "a:392;b:264;c:136", "a:128;b:128;c:64", "a:128;b:128;c:32"),   # MN / K, 4 x 3 tiles
    ("ab-ca-bc", "a:256;b:520;c:200", "a:128;b:128;c:64", "a:128;b:128;c:32"),   # K / MN, 2 x 5 tiles
    ("ab-ac-bc", "a:136;b:136;c:80", "a:128;b:128;c:48", "a:128;b:128;c:16"),    # MN / MN, ragged 2 x 2
    ("ab-ca-cb", "a:384;b:384;c:72", "a:128;b:128;c:64", "a:128;b:128;c:32"),    # K / K, 3 x 3 tiles
    ("abc-acd-db", "a:136;b:250;c:3;d:40", "a:64;c:2;b:128;d:32", "a:32;c:4;b:128;d:32"),   # 2-digit box
]


@pytest.mark.parametrize("i", range(len(PAIR_CASES)))
@pytest.mark.parametrize("dt", ["bf16", "tf32"])
def test_cta_pair(i, dt):
    expr, ext, tb, tt = PAIR_CASES[i]
    tiles = tb if dt == "bf16" else tt
    kw = dict(force_tiles=tiles, morder="X", pair=True)
    hp = tc.plan(expr, ext, dtype=dt, host_only=True, **kw)
    assert hp.info()["cta_pair"] == 1, hp.info()
    if dt == "bf16":
        check_bf16(expr, ext, seed=i, integer=True, **kw)
        check_bf16(expr, ext, seed=i, integer=False, **kw)
        check_bf16(expr, ext, seed=i + 50, integer=True, alpha=2.0, beta=1.0, **kw)
    else:
        check_f32(expr, ext, "tf32", seed=i, integer=True, **kw)
        check_f32(expr, ext, "tf32", seed=i, integer=False, **kw)
        check_f32(expr, ext, "tf32", seed=i + 50, integer=True, alpha=2.0, beta=1.0, **kw)
