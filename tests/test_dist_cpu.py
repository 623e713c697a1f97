"""Multi-process (world_size 2, gloo, CPU) tests of the sharding logic of
paper_conf_cgo_kimstkpprs19_b200/dist.py.  The per-rank compute step is
injected: the CPU oracle on the rank's slab (tests only), so the partition arithmetic, the
restricted sub-plans (host_only libtc plans) and the collectives are what is checked."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build, dist as tcdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _nd(flat, idx, ext):
    return flat.reshape([ext[c] for c in reversed(idx)])


def oracle_slab(expr, ext, index, lo, ln, A, B):
    """Compact C slab for index in [lo, lo+ln): slice the inputs, oracle on the sub-problem."""
    c, a, b = tcinputs.split_expr(expr)
    sub = dict(ext)
    sub[index] = ln

    def cut(flat, idx):
        if index not in idx:
            return flat
        arr = _nd(flat, idx, ext)
        ax = list(reversed(idx)).index(index)
        sl = [slice(None)] * arr.ndim
        sl[ax] = slice(lo, lo + ln)
        return np.ascontiguousarray(arr[tuple(sl)]).reshape(-1)

    es = ";".join(f"{k}:{v}" for k, v in sub.items())
    return oracle.contract(expr, es, cut(A, a), cut(B, b))


def _worker(rank, world, port, expr, extents, mode, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ext = tcinputs.parse_extents(extents)
    c, a, b = tcinputs.split_expr(expr)
    plan = tc.plan(expr, extents, host_only=True, fusion=False)
    # rank 0 owns the inputs; the others receive them by broadcast
    A = torch.zeros(tcinputs.numel(a, ext), dtype=torch.float64)
    B = torch.zeros(tcinputs.numel(b, ext), dtype=torch.float64)
    if rank == 0:
        A.copy_(torch.as_tensor(tcinputs.integers_np(A.numel(), 1)))
        B.copy_(torch.as_tensor(tcinputs.integers_np(B.numel(), 2)))
    try:
        if mode == "scatter":
            # the shard index is A's slowest index: rank 0 scatters A's slabs, broadcasts B
            sh = tcdist.shard_plan(plan, expr, extents, world, rank)
            assert sh.x_tensor == "A" and sh.plan is not None and sh.plan.info()["host_only"]
            nA = tcinputs.numel(a, ext)
            Aloc = A if rank == 0 else torch.zeros(tcdist.local_input_numel(sh, "A", nA, rank),
                                                   dtype=torch.float64)
            Cs = torch.zeros(sh.c_numel, dtype=torch.float64)

            def ex(p, AA, BB, CC):
                # AA is this rank's compact slab of A; the sub-problem is dense in it
                assert AA.numel() == sh.x_slabs[rank][1]
                sub = dict(ext)
                sub[sh.index] = sh.length
                es = ";".join(f"{k}:{v}" for k, v in sub.items())
                CC.copy_(torch.as_tensor(oracle.contract(expr, es, np.ascontiguousarray(AA.numpy()), BB.numpy())))
            tcdist.execute_sharded(sh, Aloc, B, Cs, execute=ex, rank=rank)
            out = [None] * world
            dist.all_gather_object(out, (sh.index, sh.lo, sh.length, Cs.numpy()))
        elif mode == "slab":
            sh = tcdist.shard_plan(plan, expr, extents, world, rank)
            Cs = torch.zeros(sh.c_numel, dtype=torch.float64)

            def ex(p, AA, BB, CC):
                assert p.info()["host_only"]
                CC.copy_(torch.as_tensor(oracle_slab(expr, ext, sh.index, sh.lo, sh.length,
                                                     AA.numpy(), BB.numpy())))
            tcdist.execute_sharded(sh, A, B, Cs, execute=ex)
            out = [None] * world
            dist.all_gather_object(out, (sh.index, sh.lo, sh.length, Cs.numpy()))
        else:
            sub, k, lo, ln = tcdist.split_k_plan(plan, expr, extents, world, rank)
            tcdist.broadcast_inputs(A, B)
            Cp = torch.zeros(tcinputs.numel(c, ext), dtype=torch.float64)

            def ex(p, AA, BB, CC):
                # partial sum over k in [lo, lo+ln): slice A and B along k
                CC.copy_(torch.as_tensor(oracle_slab_k(expr, ext, k, lo, ln, AA.numpy(), BB.numpy())))
            part = tcdist.execute_split_k(sub, A, B, Cp, world, rank, execute=ex)
            out = [None] * world
            dist.all_gather_object(out, part.numpy())
        if rank == 0:
            q.put(("ok", out))
    except Exception as e:  # pragma: no cover - surfaced through the queue
        q.put(("err", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def oracle_slab_k(expr, ext, k, lo, ln, A, B):
    c, a, b = tcinputs.split_expr(expr)
    sub = dict(ext)
    sub[k] = ln

    def cut(flat, idx):
        arr = _nd(flat, idx, ext)
        ax = list(reversed(idx)).index(k)
        sl = [slice(None)] * arr.ndim
        sl[ax] = slice(lo, lo + ln)
        return np.ascontiguousarray(arr[tuple(sl)]).reshape(-1)

    es = ";".join(f"{x}:{v}" for x, v in sub.items())
    return oracle.contract(expr, es, cut(A, a), cut(B, b))


def _run(expr, extents, mode, world=2):
    build.build()
    oracle.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, expr, extents, mode, q)) for r in range(world)]
    for p in ps:
        p.start()
    status, out = q.get(timeout=300)
    for p in ps:
        p.join(timeout=120)
    assert status == "ok", out
    return out


def test_bounds_and_shard_index():
    for n in range(1, 40):
        for w in range(1, 9):
            parts = [tcdist.bounds(n, w, r) for r in range(w)]
            assert sum(l for _, l in parts) == n
            assert max(l for _, l in parts) - min(l for _, l in parts) <= 1
            lo = 0
            for a, l in parts:
                assert a == lo
                lo += l
    assert tcdist.shard_index("abcdef-gdab-efgc", "a:4;b:4;c:4;d:4;e:4;f:4;g:4") == "f"
    assert tcdist.shard_index("abcd-aebf-dfce", "a:9;b:5;c:9;d:3;e:2;f:2") == "c"
    assert tcdist.split_k_index("ab-ac-cb", "a:4;b:4;c:9") == "c"


@pytest.mark.parametrize("expr,extents", [
    ("abcdef-gdab-efgc", "a:4;b:3;c:3;d:4;e:3;f:5;g:4"),     # shard f: C's slowest index
    ("abcd-aebf-dfce", "a:3;b:4;c:7;d:2;e:3;f:2"),            # shard c: not C's slowest
])
def test_c_slab_sharding_gloo(expr, extents):
    out = _run(expr, extents, "slab")
    ext = tcinputs.parse_extents(extents)
    c, a, b = tcinputs.split_expr(expr)
    A = tcinputs.integers_np(tcinputs.numel(a, ext), 1)
    B = tcinputs.integers_np(tcinputs.numel(b, ext), 2)
    full = oracle.contract(expr, extents, A, B)
    Cn = _nd(full, c, ext)
    s = out[0][0]
    ax = list(reversed(c)).index(s)
    pieces = [np.asarray(x[3]).reshape([ext[i] if i != s else x[2] for i in reversed(c)]) for x in out]
    assert np.array_equal(np.concatenate(pieces, axis=ax), Cn)


def test_split_k_reduce_scatter_gloo():
    expr, extents = "ab-ac-cb", "a:5;b:7;c:11"
    out = _run(expr, extents, "splitk")
    ext = tcinputs.parse_extents(extents)
    A = tcinputs.integers_np(55, 1)
    B = tcinputs.integers_np(77, 2)
    full = oracle.contract(expr, extents, A, B)
    assert np.array_equal(np.concatenate(out), full)


def test_c_slab_scatter_gloo():
    """The shard index c is A's slowest index: A travels as per-rank slabs (point-to-point),
    B by broadcast; the gathered slabs equal the oracle's C."""
    expr, extents = "abc-adc-db", "a:3;b:4;c:9;d:5"
    assert tcdist.input_slabs(expr, extents, 2, "c") == ("A", [(0, 75), (75, 60)])
    out = _run(expr, extents, "scatter")
    ext = tcinputs.parse_extents(extents)
    c, a, b = tcinputs.split_expr(expr)
    A = tcinputs.integers_np(tcinputs.numel(a, ext), 1)
    B = tcinputs.integers_np(tcinputs.numel(b, ext), 2)
    full = oracle.contract(expr, extents, A, B)
    pieces = [np.asarray(x[3]).reshape([ext[i] if i != "c" else x[2] for i in reversed(c)]) for x in out]
    assert np.array_equal(np.concatenate(pieces, axis=0), _nd(full, c, ext))


def test_partial_numel_padding():
    for n in (1, 7, 64, 1000):
        for w in (1, 2, 3, 8):
            m = tcdist.partial_numel(n, w)
            assert m % w == 0 and n <= m < n + w
