"""CPU tests of libtc's host side: the C-ABI library loads and exports every symbol of
include/libtc.h; parser / classifier against the shared rules table; fusion; planner
invariants and statistics (host_only plans: no GPU needed)."""
import ctypes
import json
import os
import re

import numpy as np
import pytest

import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build
from paper_conf_cgo_kimstkpprs19_b200.csrc_variants import BF16_VARIANTS

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def _built():
    build.build()


def test_exports_every_header_symbol():
    hdr = open(os.path.join(ROOT, "include", "libtc.h")).read()
    names = set(re.findall(r"\b(tc_[a-z_]+)\s*\(", hdr))
    assert len(names) >= 14
    L = ctypes.CDLL(build.SO)
    for n in sorted(names):
        assert hasattr(L, n), n


def test_validation_rules_golden():
    rules = json.load(open(os.path.join(ROOT, "tests", "golden", "validation_rules.json")))["rules"]
    for expr, extents, want in rules:
        assert tc.check(expr, extents) == want, (expr, extents)


def test_classification_eq1_and_bracket_form():
    a = tc.plan("abcd-aebf-dfce", tcinputs.EQ1_EXTENTS, host_only=True).info()
    b = tc.plan("C[a,b,c,d] = A[a,e,b,f] * B[d,f,c,e]", tcinputs.EQ1_EXTENTS, host_only=True).info()
    cls = {x["name"]: x["cls"] for x in a["indices"]}
    assert cls == {"a": "extA", "b": "extA", "c": "extB", "d": "extB", "e": "int", "f": "int"}
    assert a["X"] == "A"          # C's FVI a lives in A
    for k in ("indices", "m", "n", "k", "variant", "Mt", "Nt", "Kt", "nctas", "nsteps"):
        assert a[k] == b[k], k


def test_fusion_row_a2():
    i = tc.plan("abcd-ea-ebcd", "a:72;b:72;c:72;d:72;e:72", host_only=True).info()
    assert sorted(x["name"] for x in i["indices"]) == ["a", "b*c*d", "e"]
    i = tc.plan("abcd-abef-efcd", ";".join(f"{c}:8" for c in "abcdef"), host_only=True).info()
    assert sorted(x["name"] for x in i["indices"]) == ["a*b", "c*d", "e*f"]   # a pure GEMM
    i = tc.plan("abcd-aebf-dfce", "a:1;b:5;c:6;d:7;e:2;f:3", host_only=True).info()
    assert "a" not in [x["name"] for x in i["indices"]]                        # extent 1 dropped
    i = tc.plan("abcd-ea-ebcd", "a:72;b:72;c:72;d:72;e:72", host_only=True, fusion=False).info()
    assert len(i["indices"]) == 5


@pytest.mark.parametrize("dtype", ["f64", "bf16"])
@pytest.mark.parametrize("cost", ["b200", "paper"])
def test_planner_invariants_tccg(cost, dtype):
    for case in [tcinputs.eq1()] + tcinputs.tccg48():
        i = tc.plan(case.expr, case.extents, host_only=True, cost=cost, dtype=dtype).info()
        assert i["dtype"] == dtype
        assert (i["variant"] in BF16_VARIANTS) == (dtype == "bf16")
        assert i["vecX"] <= (8 if dtype == "bf16" else 2) and i["vecY"] <= (8 if dtype == "bf16" else 2)
        assert i["Mt"] <= i["BM"] and i["Nt"] <= i["BN"] and i["Kt"] <= i["BK"]
        for x in i["indices"]:
            assert 1 <= x["tile"] <= x["n"]
        assert i["flops_padded"] >= i["flops"] * (1 - 1e-12)
        assert i["stats"]["plan_ms"] < 1000   # host-side sanity bound, not a perf claim
        # every index is on exactly one side (an index maps to one dimension)
        names = i["m"] + i["n"] + i["k"]
        assert sorted(names) == sorted(x["name"] for x in i["indices"])


def test_paper_mode_eq1_config_space():
    # SURVEY 8(a) worked fixture: eq. (1) at N = 16 with the V100 value sets of P:L176:
    # TB_x {a:4|8|16} x REG_x {b:2|4|6|8} x TB_y {d:4|8|16} x REG_y {c:2|4|6|8}
    # x TB_k {e:4|8|16 or f:4|8|16} = 3*4*3*4*6 = 864 raw configurations.
    i = tc.plan("abcd-aebf-dfce", tcinputs.EQ1_EXTENTS, host_only=True, cost="paper").info()
    assert i["stats"]["raw"] == 864
    assert i["stats"]["pruned"] + i["stats"]["ranked"] == 864
    assert i["stats"]["pruned"] > 0
    assert i["paper_mapping"].startswith("TB_x=[a:")


def test_forced_fig3_config():
    # Fig. 3: N = 16, T_a = 16, T_e = 1, T_b = 4, T_f = 16, T_d = 4.
    i = tc.plan("abcd-aebf-dfce", tcinputs.EQ1_EXTENTS, host_only=True,
                force_tiles="a:16;e:1;b:4;f:16;d:4;c:1").info()
    t = {x["name"]: x["tile"] for x in i["indices"]}
    assert t == {"a": 16, "b": 4, "c": 1, "d": 4, "e": 1, "f": 16}
    assert i["Mt"] == 64 and i["Nt"] == 4 and i["Kt"] == 16
    assert i["nctas"] == 1 * 4 * 16 * 4 and i["nsteps"] == 16


def test_forced_fig2_config():
    # Fig. 2: T_a = T_b = T_c = T_d = 2 -> 16 C elements per thread block.
    i = tc.plan("abcd-aebf-dfce", "a:2;b:2;c:2;d:2;e:2;f:2", host_only=True,
                force_tiles="a:2;b:2;c:2;d:2;e:2;f:2").info()
    assert i["Mt"] * i["Nt"] == 16 and i["nctas"] == 1


def test_restrict_offsets_and_extents():
    p = tc.plan("abcdef-gdab-efgc", "a:8;b:4;c:4;d:8;e:4;f:6;g:8", host_only=True, fusion=False)
    s = p.restrict("f", 2, 3)
    i = s.info()
    assert {x["name"]: x["n"] for x in i["indices"]}["f"] == 3
    # f is C's slowest index: C base = 2 * stride_C(f) = 2 * 8*4*4*8*4
    assert i["tensors"]["C"]["base"] == 2 * 8 * 4 * 4 * 8 * 4
    assert i["tensors"]["B"]["base"] == 2 * 4      # B = efgc: stride(f) = N_e
    s2 = p.restrict("f", 2, 3, tc.SLAB_C)
    assert s2.info()["tensors"]["C"]["base"] == 0
    k = p.restrict("g", 0, 4)                      # split-K slab of the internal index
    assert {x["name"]: x["n"] for x in k.info()["indices"]}["g"] == 4
    with pytest.raises(tc.TcError):
        p.restrict("f", 5, 3)
    with pytest.raises(tc.TcError):
        p.restrict("z", 0, 1)


def test_plan_is_deterministic():
    a = tc.plan("abcd-aebf-fdec", ";".join(f"{c}:72" for c in "abcdef"), host_only=True).info()
    b = tc.plan("abcd-aebf-fdec", ";".join(f"{c}:72" for c in "abcdef"), host_only=True).info()
    a["stats"].pop("plan_ms"); b["stats"].pop("plan_ms")
    assert a == b


def test_errors_are_status_codes():
    with pytest.raises(tc.TcError) as e:
        tc.plan("abcd-aebf-dfc", "a:2;b:2;c:2;d:2;e:2;f:2", host_only=True)
    assert e.value.status == "TC_ERR_INDEX" and "exactly two" in e.value.detail
    import ctypes
    h = ctypes.c_void_p()
    st = tc.lib().tc_plan(ctypes.byref(h), b"ab-ac-cb", b"a:2;b:2;c:2", 7)   # no such dtype
    assert tc.lib().tc_status_string(st).decode() == "TC_ERR_UNSUPPORTED" and not h.value
    for dt in ("f32", "tf32", "bf16"):                 # every dtype of the header is built
        assert tc.plan("ab-ac-cb", "a:2;b:2;c:2", dtype=dt, host_only=True).info()["dtype"] == dt
    with pytest.raises(tc.TcError) as e:              # a BF16 variant for a TF32 plan
        tc.plan("ab-ac-cb", "a:2;b:2;c:2", dtype="tf32", host_only=True, variant=11)
    assert e.value.status == "TC_ERR_INVALID_ARG"
    with pytest.raises(tc.TcError) as e:              # an FP64 variant for a BF16 plan
        tc.plan("ab-ac-cb", "a:2;b:2;c:2", dtype="bf16", host_only=True, variant=0)
    assert e.value.status == "TC_ERR_INVALID_ARG"
    p = tc.plan("ab-ac-cb", "a:2;b:2;c:2", host_only=True)
    with pytest.raises(tc.TcError) as e:
        p.execute_ptr(16, 32, 64)
    assert e.value.status == "TC_ERR_CUDA"          # host_only plans cannot execute


def test_plan_cache_reuse_and_refcounts():
    # NEXT-1: plan once, run many — same arguments => the same plan object
    tc.plan_cache_clear()
    e, x = "abcd-aebf-dfce", "a:24;b:16;c:24;d:16;e:16;f:24"
    p1 = tc.plan_cached(e, x, host_only=True)
    p2 = tc.plan_cached(e, x, host_only=True)
    assert p1.handle.value == p2.handle.value and tc.plan_cache_size() == 1
    p3 = tc.plan_cached(e, x, dtype="bf16", host_only=True)        # another key
    p4 = tc.plan_cached(e, x, host_only=True, variant=3)
    assert len({p1.handle.value, p3.handle.value, p4.handle.value}) == 3 and tc.plan_cache_size() == 3
    assert p1.info() == tc.plan(e, x, host_only=True).info() | {"stats": p1.info()["stats"]}
    # dropping every Python handle and the cache frees nothing twice; live handles stay valid
    del p2
    tc.plan_cache_clear()
    assert tc.plan_cache_size() == 0 and p1.info()["dtype"] == "f64" and p3.info()["dtype"] == "bf16"
    # failures are not cached
    with pytest.raises(tc.TcError):
        tc.plan_cached("ab-ac-cd", "a:2;b:2;c:2;d:2", host_only=True)
    assert tc.plan_cache_size() == 0


def test_batch_index_classification_and_limits():
    # an index of C, A and B is a batch (Hadamard) index: neither m, n nor k (R31)
    i = tc.plan("abcd-aebd-ecd", "a:24;b:6;c:40;d:3;e:50", host_only=True).info()
    cls = {d["name"]: d["cls"] for d in i["indices"]}
    assert cls == {"a": "extA", "b": "extA", "c": "extB", "d": "batch", "e": "int"}
    assert "d" not in i["m"] + i["n"] + i["k"] and i["nbatch"] == 3
    assert tc.plan("ab-ab-ab", "a:5;b:7", host_only=True).info()["nbatch"] == 35
    with pytest.raises(tc.TcError) as e:                       # > 65535 batch slabs
        tc.plan("abc-abc-abc", "a:100;b:100;c:10", host_only=True)
    assert e.value.status == "TC_ERR_UNSUPPORTED"
    with pytest.raises(tc.TcError) as e:                       # > 4 batch indices
        tc.plan("abcde-abcde-abcde", "a:2;b:2;c:2;d:2;e:2", host_only=True)
    assert e.value.status == "TC_ERR_UNSUPPORTED"


def test_execute_group_validation_host():
    """tc_execute_group checks, before any launch, that every member gives C the same layout
    (SURVEY 8(f) NEXT-4): the 18 CCSD(T) triples pass validation and reach tc_execute (which
    refuses host_only plans with TC_ERR_CUDA); a member with another C layout is refused with
    TC_ERR_INVALID_ARG; so are n < 1 and a dtype mismatch."""
    ext = "a:6;b:5;c:7;d:6;e:5;f:7;g:9"
    exprs = [c.expr for c in tcinputs.tccg48() if c.group.startswith("CCSDT")]
    plans = [tc.plan(e, ext, host_only=True) for e in exprs]
    big = 1 << 40
    A = [big + i * (1 << 30) for i in range(len(plans))]
    B = [2 * big + i * (1 << 30) for i in range(len(plans))]
    C = 3 * big
    with pytest.raises(tc.TcError) as e:
        tc.execute_group_ptr(plans, A, B, C)
    assert e.value.status == "TC_ERR_CUDA"                                  # reached tc_execute
    other = tc.plan("abcdef-gdab-efgc", "a:6;b:5;c:7;d:6;e:5;f:8;g:9", host_only=True)
    for bad in (plans + [other], [other] + plans[:2]):
        with pytest.raises(tc.TcError) as e:
            tc.execute_group_ptr(bad, A[:len(bad)] + [big] * (len(bad) - len(A)),
                                 B[:len(bad)] + [big] * (len(bad) - len(B)), C)
        assert e.value.status == "TC_ERR_INVALID_ARG"
    perm = tc.plan("bacdef-gdab-efgc", ext, host_only=True)
    with pytest.raises(tc.TcError) as e:                           # C positions permuted
        tc.execute_group_ptr([plans[0], perm], A[:2], B[:2], C)    
    assert e.value.status == "TC_ERR_INVALID_ARG"
    f32 = tc.plan(exprs[0], ext, dtype="f32", host_only=True)
    with pytest.raises(tc.TcError) as e:
        tc.execute_group_ptr([plans[0], f32], A[:2], B[:2], C)
    assert e.value.status == "TC_ERR_INVALID_ARG"
    with pytest.raises(tc.TcError) as e:
        tc.execute_group_ptr([], [], [], C)
    assert e.value.status == "TC_ERR_INVALID_ARG"


def test_plan_tuned_beta_errors_host():
    """tc_plan_tuned_beta validates like tc_plan_tuned: NULL tensors / topk < 1 are
    TC_ERR_INVALID_ARG, a host_only plan is TC_ERR_CUDA; *tuned stays NULL."""
    p = tc.plan("abcdef-gdab-efgc", "a:6;b:5;c:7;d:6;e:5;f:7;g:9", host_only=True)
    L = tc.lib()
    h = ctypes.c_void_p()
    x = ctypes.c_void_p(1 << 40)
    assert L.tc_plan_tuned_beta(ctypes.byref(h), p._h, None, x, x, 2, 1, 1.0, None) == 1
    assert L.tc_plan_tuned_beta(ctypes.byref(h), p._h, x, x, x, 0, 1, 1.0, None) == 7   # host_only first
    assert not h.value


def test_reserved_opts_rejected_and_restrict_overflow():
    """tc_plan_opts.reserved[] must be zero (no hidden switches reach the kernels); a slab
    whose begin + len would overflow int64 is TC_ERR_EXTENT, not an out-of-bounds plan."""
    o = tc._opts("b200", True, None, None, True, False, None)
    o.reserved[0] = 64
    h = ctypes.c_void_p()
    st = tc.lib().tc_plan_ex(ctypes.byref(h), b"ab-ac-cb", b"a:8;b:8;c:8", 0, ctypes.byref(o))
    assert tc.STATUS[st] == "TC_ERR_INVALID_ARG" and not h.value
    p = tc.plan("ab-ac-cb", "a:8;b:8;c:8", host_only=True)
    for begin, length in (((1 << 63) - 2, 4), (7, 2), (-1, 1), (0, 0)):
        with pytest.raises(tc.TcError) as e:
            p.restrict("a", begin, length)
        assert e.value.status == "TC_ERR_EXTENT"


def test_paper_mode_lists_tuning_candidates():
    """Paper-mode plans carry the B200-ranked per-variant candidates too, so measured tuning
    (tc_plan_tuned) has more than the planned variant to time in either cost mode."""
    for ext in ("a:16;b:16;c:16;d:16;e:16;f:16", "a:2;b:2;c:2;d:2;e:2;f:2"):   # (2: paper sets prune all)
        i = tc.plan("abcd-aebf-dfce", ext, cost="paper", host_only=True).info()
        pv = i["stats"]["per_variant"]
        assert len(pv) >= 2 and [t for _, t in pv] == sorted(t for _, t in pv)


def test_group_plan_triples_host():
    """Fused group planning (NEXT-4) of the 18 CCSD(T) triples without a GPU: one 4^6 C tile
    makes every member a 64 x 64 DMMA tile (3 C indices per operand), BK follows the internal
    extent, and the simulated flush of every member into the swizzled box is conflict-free
    (4 warps x 32 accesses x load+store x 2 wavefronts = 512)."""
    exprs = [c.expr for c in tcinputs.tccg48() if c.group.startswith("CCSDT")]
    for ext, bk in (("a:24;b:16;c:16;d:24;e:16;f:16;g:24", 24), (";".join(f"{x}:16" for x in "abcdefg"), 16)):
        g = tc.plan_group([tc.plan(e, ext, host_only=True) for e in exprs])
        i = g.info()
        assert i["T"] == [4] * 6 and i["BK"] == bk and i["box"] == 4096
        assert all(m["Mt"] == 64 and m["Nt"] == 64 and m["nsteps"] == 1 for m in i["per_member"])
        assert all(m["flush_wf"] == 512 for m in i["per_member"])
        # FVI runs: 16-B vectors on both operands of every member (aligned extents)
        assert all(m["vecX"] == 2 and m["vecY"] == 2 for m in i["per_member"])
        with pytest.raises(tc.TcError) as e:                     # planned, not executable
            g.execute_ptr([1 << 40] * 18, [1 << 41] * 18, 1 << 42)
        assert e.value.status == "TC_ERR_CUDA"


def test_group_plan_errors_host():
    ext = "a:6;b:5;c:7;d:6;e:5;f:7;g:9"
    p = tc.plan("abcdef-gdab-efgc", ext, host_only=True)
    with pytest.raises(tc.TcError) as e:
        tc.plan_group([])
    assert e.value.status == "TC_ERR_INVALID_ARG"
    with pytest.raises(tc.TcError) as e:                         # C laid out differently
        tc.plan_group([p, tc.plan("abcdef-gdab-efgc", "a:6;b:5;c:7;d:6;e:5;f:8;g:9", host_only=True)])
    assert e.value.status == "TC_ERR_INVALID_ARG"
    with pytest.raises(tc.TcError) as e:                         # batch index
        tc.plan_group([tc.plan("abc-abd-cbd", "a:4;b:4;c:4;d:4", host_only=True)])
    assert e.value.status == "TC_ERR_UNSUPPORTED"
    with pytest.raises(tc.TcError) as e:                         # an operand of rank 9 (> 8)
        tc.plan_group([tc.plan("abcdefgh-abcdefghi-i", ";".join(f"{x}:2" for x in "abcdefghi"), host_only=True)])
    assert e.value.status == "TC_ERR_UNSUPPORTED"


def test_plan_strided_validation_and_span():
    """tc_plan_strided (row f3): stride checks, spans, fusion only over contiguous strides."""
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    # explicit dense strides plan exactly like tc_plan
    d = tc.plan("abcd-aebf-dfce", "a:12;b:10;c:9;d:8;e:7;f:6", host_only=True).info()
    s = tc.plan_strided("abcd-aebf-dfce", "a:12;b:10;c:9;d:8;e:7;f:6",
                        {"C": [1, 12, 120, 1080], "A": [1, 12, 84, 840], "B": [1, 8, 48, 336]}, host_only=True).info()
    assert [x["tile"] for x in d["indices"]] == [x["tile"] for x in s["indices"]]
    # a padded pitch: spans grow, numel does not; a and c of ab-ac-cb no longer fuse with b
    p = tc.plan_strided("ab-ac-cb", "a:70;b:50;c:40", {"C": [1, 72], "A": [1, 80]}, host_only=True)
    assert p.numel("C") == 70 * 50 and p.span("C") == 69 + 49 * 72 + 1
    assert p.span("A") == 69 + 39 * 80 + 1 and p.span("B") == 40 * 50
    # fusion: the a-b run fuses only when its strides are contiguous in every tensor
    q = tc.plan("abc-abd-dc", "a:4;b:5;c:6;d:7", host_only=True).info()
    qs = tc.plan_strided("abc-abd-dc", "a:4;b:5;c:6;d:7", {"C": [1, 5, 25], "A": [1, 4, 20]},
                         host_only=True).info()
    assert any("*" in x["name"] for x in q["indices"])          # a*b fused when dense
    assert not any("*" in x["name"] for x in qs["indices"])     # C's a-b pitch 5 != 4: kept apart
    for bad in ({"C": [1, 3]}, {"C": [0, 70]}, {"A": [-1, 70]}, {"C": [1, 1 << 61]}):
        with pytest.raises(tc.TcError) as e:
            tc.plan_strided("ab-ac-cb", "a:5;b:7;c:3", bad, host_only=True)
        assert e.value.status == "TC_ERR_INVALID_ARG", bad


def test_resize_and_select_host():
    """Representative-size plans (row f1): tiles clamp, the variant stays, a structure change
    (an extent-1 index) re-plans, selection follows the cost model, strided plans refuse."""
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    expr = "abcd-aebf-dfce"
    rep = tc.plan(expr, "a:16;b:16;c:16;d:16;e:16;f:16", host_only=True)
    ri = rep.info()
    s = rep.resize("a:5;b:40;c:7;d:3;e:9;f:70").info()
    assert s["resized"] == 1 and s["variant"] == ri["variant"]
    ext = dict(a=5, b=40, c=7, d=3, e=9, f=70)
    for x, y in zip(ri["indices"], s["indices"]):
        assert x["name"] == y["name"] and y["tile"] == min(x["tile"], ext[x["name"]])
    assert rep.resize("a:1;b:16;c:16;d:16;e:16;f:16").info()["resized"] == 0
    vs = [tc.plan(expr, f"a:{n};b:{n};c:{n};d:{n};e:{n};f:{n}", host_only=True) for n in (8, 16, 72)]
    big = "a:64;b:64;c:64;d:64;e:64;f:64"
    p, ch = tc.select(vs, big)
    preds = [v.resize(big).info()["t_pred_ms"] for v in vs]
    assert ch == int(np.argmin(preds)) and p.info()["t_pred_ms"] == min(preds)
    st = tc.plan_strided("ab-ac-cb", "a:5;b:7;c:3", {"C": [1, 8]}, host_only=True)
    with pytest.raises(tc.TcError) as e:
        st.resize("a:6;b:7;c:3")
    assert e.value.status == "TC_ERR_INVALID_ARG"


def test_large_index_splitting_and_fusion_cap():
    """Row f1: an index longer than 2^31-1 is split into two exact factors; fusion
    never builds an index past 2^31-1; a prime extent past 2^31 is unsupported."""
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    n = 3 << 30                                  # 3 * 2^30 > 2^31 - 1
    i = tc.plan("ab-a-b", f"a:{n};b:3", host_only=True).info()
    ext = {x["name"]: x["n"] for x in i["indices"]}
    assert ext == {"a": n // 2, "a'": 2, "b": 3}
    assert i["tensors"]["A"]["stride"] == [1, n // 2] and i["tensors"]["C"]["stride"][:2] == [1, n // 2]
    # fusion cap: a and b would fuse into 2.5e9 elements
    j = tc.plan("abc-abd-dc", "a:50000;b:50000;c:1;d:1", host_only=True).info()
    assert sorted(x["name"] for x in j["indices"]) == ["a", "b"]
    with pytest.raises(tc.TcError) as e:
        tc.plan("ab-a-b", "a:2147483659;b:2", host_only=True)   # a prime past 2^31
    assert e.value.status == "TC_ERR_UNSUPPORTED"


def test_cta_pair_needs_c_fvi_leading_m():
    """CTA-pair instances store straight from TMEM rows (no epilogue staging, a sixth stage):
    a plan whose C runs need the CTA-wide staged pass (C's FVI an inner m digit) stays
    single-CTA even when pairs are asked for; the GEMM-like layout pairs."""
    from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
    i = tc.plan("abcd-ebad-ce", "a:32;b:4;c:128;d:8;e:64", dtype="bf16", force_tiles="b:2;a:16;d:4;c:128;e:64",
                morder="X", pair=True, host_only=True).info()
    assert i["tma_operands"] == 1 and i["vecC"] == 8 and i["cs0"] > 1 and i["cta_pair"] == 0
    j = tc.plan("ab-ac-cb", "a:392;b:264;c:136", dtype="bf16", force_tiles="a:128;b:128;c:64", pair=True,
                host_only=True).info()
    assert j["cs0"] == 1 and j["cta_pair"] == 1


def test_stream_path_planning():
    """The streaming BF16 path (stream.hpp): planned for the memory-bound tensor x matrix TCCG
    cases #1-8 (both row modes), never for other dtypes, batch indices, large Y-side extents or
    when the options turn it off; tiles are TMA-legal boxes and the units fit the 8 warps."""
    import tcinputs
    for c in tcinputs.tccg48():
        s = tc.plan(c.expr, c.extents, "bf16", host_only=True).info()["stream"]
        if c.id <= 8:
            assert s["on"] == 1, (c.id, s)
            assert s["mode"] == ("K" if c.id in (7, 8) else "T")
            assert 1 <= s["units"] <= 8 and s["AR"] in (4, 8) and s["KB"] % 16 == 0
            assert all(t <= 256 for t in s["tiles"].values())
            assert s["smem"] <= (115712 if s["AR"] == 4 else 232448)
        else:
            assert s["on"] == 0, (c.id, s)
    c1 = tcinputs.tccg48()[0]
    # FP32 storage (TF32 / split FP32): streaming shapes; by default in SM_T only
    for dt in ("f32", "tf32"):
        for c in tcinputs.tccg48()[:8]:
            s = tc.plan(c.expr, c.extents, dt, host_only=True).info()["stream"]
            assert s["on"] == 1 and s["active"] == (0 if c.id in (7, 8) else 1), (dt, c.id, s)
    # FP64: streaming shapes too; used by default below 0.8 of the DMMA ridge (#6 / #8, K = 312,
    # sit at the ridge: the tile kernel by default, tuning times both)
    for c in tcinputs.tccg48()[:8]:
        s = tc.plan(c.expr, c.extents, "f64", host_only=True).info()["stream"]
        assert s["on"] == 1 and s["active"] == (0 if c.id in (6, 8) else 1), (c.id, s)
    assert tc.plan(c1.expr, c1.extents, "bf16", host_only=True, stream=False).info()["stream"]["on"] == 0
    # a forced variant keeps the path off unless asked for
    assert tc.plan(c1.expr, c1.extents, "bf16", host_only=True, variant=11).info()["stream"]["on"] == 0
    assert tc.plan(c1.expr, c1.extents, "bf16", host_only=True, variant=11, stream=True).info()["stream"]["on"] == 1
    # batch index, Y-side extent above 32, X's FVI = C's FVI: not streaming shapes
    assert tc.plan("abh-ach-cbh", "a:16;b:16;c:16;h:4", "bf16", host_only=True).info()["stream"]["on"] == 0
    assert tc.plan("abc-bda-dc", "a:16;b:16;c:40;d:16", "bf16", host_only=True).info()["stream"]["on"] == 0
    assert tc.plan("abc-adb-dc", "a:16;b:16;c:16;d:16", "bf16", host_only=True).info()["stream"]["on"] == 0
