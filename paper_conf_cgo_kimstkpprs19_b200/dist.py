"""Multi-GPU execution of libtc contractions; one process per GPU.

* C-slab sharding (the default): the largest external index s of C (ties: the rightmost,
  i.e. slowest, so a rank's slab of C is contiguous) is split into balanced ranges; rank r
  computes C[..., s in [lo_r, hi_r), ...] with ``tc_plan_restrict`` and a compact C slab
  (TC_SLAB_C).  No reduction is needed; the one exchange step is the distribution of the
  inputs (``broadcast_inputs``: NCCL broadcast over NVLink from the root).
* split-K: for contractions whose external space is too small to fill p x 148 SMs, the
  largest internal index is split; each rank computes a full-size partial C and the
  partials are summed with a reduce-scatter (NCCL), leaving |C|/p elements per rank.

torch.distributed is the plumbing (process group, NCCL collectives); every FLOP runs in
libtc's kernels.  The partition arithmetic is pure Python and is tested with the gloo
backend on CPU (tests/test_dist_cpu.py).
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist

from . import binding as tc


def _parse(expr: str):
    c, a, b = expr.split("-")
    return c, a, b


def _extents(extents: str) -> dict:
    out = {}
    for part in extents.split(";"):
        part = part.strip()
        if part:
            k, v = part.split(":")
            out[k.strip()] = int(v)
    return out


def shard_index(expr: str, extents: str) -> str:
    """argmax_{i in ext(C)} N_i; ties go to the rightmost (slowest) index of C."""
    c, _, _ = _parse(expr)
    ext = _extents(extents)
    best = None
    for i in c:
        if best is None or ext[i] >= ext[best]:
            best = i
    return best


def split_k_index(expr: str, extents: str) -> str:
    """The largest internal index (ties: rightmost in A)."""
    c, a, _ = _parse(expr)
    ext = _extents(extents)
    best = None
    for i in a:
        if i not in c and (best is None or ext[i] >= ext[best]):
            best = i
    if best is None:
        raise ValueError("no internal index to split")
    return best


def bounds(n: int, world: int, rank: int) -> tuple[int, int]:
    """Balanced [lo, lo + len) of range(n) for rank; sizes differ by at most one."""
    q, r = divmod(n, world)
    lo = rank * q + min(rank, r)
    return lo, q + (1 if rank < r else 0)


@dataclass
class Shard:
    index: str
    lo: int
    length: int
    plan: "tc.Plan | None"      # restricted plan (None if this rank owns nothing)
    c_numel: int                # elements of this rank's compact C slab
    c_contiguous: bool          # the slab is a contiguous range of the full C
    c_offset: int               # its first element in the full C (if contiguous)


def shard_plan(plan: "tc.Plan", expr: str, extents: str, world: int, rank: int,
               index: str | None = None) -> Shard:
    """Rank `rank`'s C-slab sub-plan (compact C slab, inputs addressed in the full tensors)."""
    s = index or shard_index(expr, extents)
    ext = _extents(extents)
    lo, ln = bounds(ext[s], world, rank)
    c, _, _ = _parse(expr)
    per = 1
    for i in c:
        per *= ext[i] if i != s else ln
    contiguous = c[-1] == s or all(ext[i] == 1 for i in c[c.index(s) + 1:])
    stride = 1
    for i in c[:c.index(s)]:
        stride *= ext[i]
    sub = plan.restrict(s, lo, ln, tc.SLAB_C) if ln > 0 else None
    return Shard(s, lo, ln, sub, per if ln > 0 else 0, contiguous, lo * stride)


def broadcast_inputs(A: torch.Tensor, B: torch.Tensor, src: int = 0, group=None):
    """Distribute the inputs from `src` to every rank (NCCL broadcast over NVLink)."""
    dist.broadcast(A, src, group=group)
    dist.broadcast(B, src, group=group)


def execute_sharded(shard: Shard, A, B, C_slab, alpha=1.0, beta=0.0, src: int = 0,
                    distribute: bool = True, execute=None):
    """Broadcast the inputs, then compute this rank's C slab.  `execute(plan, A, B, C)` may
    be injected (CPU tests); by default it is libtc's tc_execute."""
    if distribute:
        broadcast_inputs(A, B, src)
    if shard.plan is not None:
        (execute or (lambda p, a, b, c: p.execute(a, b, c, alpha, beta)))(shard.plan, A, B, C_slab)
    return C_slab


def split_k_plan(plan: "tc.Plan", expr: str, extents: str, world: int, rank: int,
                 index: str | None = None):
    k = index or split_k_index(expr, extents)
    ext = _extents(extents)
    lo, ln = bounds(ext[k], world, rank)
    return (plan.restrict(k, lo, ln) if ln > 0 else None), k, lo, ln


def reduce_scatter_sum(partial: torch.Tensor, world: int, rank: int, group=None) -> torch.Tensor:
    """Sum the full-size partial C's of all ranks and keep this rank's contiguous |C|/p part
    (balanced bounds).  NCCL: one reduce-scatter; other backends: all-reduce + slice."""
    n = partial.numel()
    chunk = -(-n // world)
    if dist.get_backend(group) == "nccl":
        padded = partial if n == chunk * world else torch.cat(
            [partial, partial.new_zeros(chunk * world - n)])
        out = partial.new_empty(chunk)
        dist.reduce_scatter_tensor(out, padded, op=dist.ReduceOp.SUM, group=group)
        lo = rank * chunk
        return out[:max(0, min(chunk, n - lo))]
    full = partial.clone()
    dist.all_reduce(full, op=dist.ReduceOp.SUM, group=group)
    lo = rank * chunk
    return full[lo:min(n, lo + chunk)]


def execute_split_k(sub, A, B, C_partial, world, rank, alpha=1.0, beta=0.0, execute=None,
                    group=None):
    """Each rank: partial C over its k-range (beta applied on rank 0 only), then the
    reduce-scatter.  Returns this rank's |C|/p chunk of the summed result."""
    if rank != 0:
        C_partial.zero_()
    b = beta if rank == 0 else 0.0
    if sub is not None:
        (execute or (lambda p, a, bb, c: p.execute(a, bb, c, alpha, b)))(sub, A, B, C_partial)
    elif rank == 0 and beta != 1.0:
        C_partial.mul_(beta)
    return reduce_scatter_sum(C_partial, world, rank, group)
