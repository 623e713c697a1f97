"""Multi-GPU execution of libtc contractions; one process per GPU.

* C-slab sharding (the default): the largest external index s of C (ties: the rightmost,
  i.e. slowest, so a rank's slab of C is contiguous) is split into balanced ranges; rank r
  computes C[..., s in [lo_r, hi_r), ...] with ``tc_plan_restrict`` and a compact C slab
  (TC_SLAB_C).  No reduction is needed; the one exchange step is the distribution of the
  inputs (``distribute_inputs``): the input holding s is SCATTERED when s is its slowest
  index (each rank receives only its contiguous slab, TC_SLAB_A / TC_SLAB_B: batched NCCL
  send/recv over NVLink), the other input is broadcast.
* split-K: for contractions whose external space is too small to fill p x 148 SMs, the
  largest internal index is split; each rank computes a full-size partial C and the
  partials are summed with a reduce-scatter (NCCL), leaving |C|/p elements per rank.
  Partials keep the accumulator precision: BF16 plans write FP32 partials (plan option
  out_f32), reduced in FP32 and rounded once (libtc tc_round_bf16); FP64 stays FP64.

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
    x_tensor: "str | None" = None   # "A" / "B": the input scattered as compact slabs
    x_slabs: "list | None" = None   # (offset, numel) of every rank's slab of that input


def input_slabs(expr: str, extents: str, world: int, index: str):
    """The input holding shard index `index`, when `index` is its slowest non-trivial index
    (so each rank's slab of it is one contiguous range): (name, [(offset, numel)] per rank).
    None otherwise (the input is then broadcast whole)."""
    c, a, b = _parse(expr)
    ext = _extents(extents)
    for name, idx in (("A", a), ("B", b)):
        if index in idx:
            p = idx.index(index)
            if any(ext[i] != 1 for i in idx[p + 1:]):
                return None
            stride = 1
            for i in idx[:p]:
                stride *= ext[i]
            out = []
            for r in range(world):
                lo, ln = bounds(ext[index], world, r)
                out.append((lo * stride, ln * stride))
            return name, out
    return None


def shard_plan(plan: "tc.Plan", expr: str, extents: str, world: int, rank: int,
               index: str | None = None, scatter: bool = True) -> Shard:
    """Rank `rank`'s C-slab sub-plan: compact C slab; the input holding the shard index as a
    compact slab too when it can be scattered (``input_slabs``), the other input addressed in
    the full tensor."""
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
    xs = input_slabs(expr, extents, world, s) if scatter else None
    flags = tc.SLAB_C | ({"A": tc.SLAB_A, "B": tc.SLAB_B}[xs[0]] if xs else 0)
    sub = plan.restrict(s, lo, ln, flags) if ln > 0 else None
    return Shard(s, lo, ln, sub, per if ln > 0 else 0, contiguous, lo * stride,
                 xs[0] if xs else None, xs[1] if xs else None)


def local_input_numel(shard: Shard, name: str, full_numel: int, rank: int) -> int:
    """Elements this rank holds of input `name` ("A" / "B"): its slab if scattered."""
    if shard.x_tensor == name:
        return shard.x_slabs[rank][1]
    return full_numel


def distribute_inputs(shard: Shard, A: torch.Tensor, B: torch.Tensor, rank: int, src: int = 0, group=None):
    """The one exchange step of C-slab sharding.  The scattered input (if any): `src` holds it
    whole and sends every other rank its slab (batched point-to-point, NCCL over NVLink);
    the others hold a slab-sized buffer.  Every other input is broadcast from `src`."""
    for name, T in (("A", A), ("B", B)):
        if shard.x_tensor != name:
            dist.broadcast(T, src, group=group)
    if shard.x_tensor is None:
        return
    T = A if shard.x_tensor == "A" else B
    ops = []
    if rank == src:
        for r, (off, n) in enumerate(shard.x_slabs):
            if r != src and n > 0:
                ops.append(dist.P2POp(dist.isend, T.narrow(0, off, n), r, group=group))
    elif shard.x_slabs[rank][1] > 0:
        ops.append(dist.P2POp(dist.irecv, T, src, group=group))
    if ops:
        for req in dist.batch_isend_irecv(ops):
            req.wait()


def local_operands(shard: Shard, A: torch.Tensor, B: torch.Tensor, rank: int, src: int = 0):
    """The (A, B) the rank's sub-plan reads: on `src` the scattered input is its own slab of
    the whole tensor (a contiguous view)."""
    if shard.x_tensor is None or rank != src:
        return A, B
    off, n = shard.x_slabs[rank]
    if shard.x_tensor == "A":
        return A.narrow(0, off, n), B
    return A, B.narrow(0, off, n)


def broadcast_inputs(A: torch.Tensor, B: torch.Tensor, src: int = 0, group=None):
    """Distribute the inputs from `src` to every rank (NCCL broadcast over NVLink)."""
    dist.broadcast(A, src, group=group)
    dist.broadcast(B, src, group=group)


def execute_sharded(shard: Shard, A, B, C_slab, alpha=1.0, beta=0.0, src: int = 0,
                    distribute: bool = True, execute=None, rank: int | None = None):
    """Distribute the inputs (scatter / broadcast), then compute this rank's C slab.
    `execute(plan, A, B, C)` may be injected (CPU tests); by default it is libtc's tc_execute."""
    rank = dist.get_rank() if rank is None else rank
    if distribute:
        distribute_inputs(shard, A, B, rank, src)
    if shard.plan is not None:
        a, b = local_operands(shard, A, B, rank, src)
        (execute or (lambda p, x, y, c: p.execute(x, y, c, alpha, beta)))(shard.plan, a, b, C_slab)
    return C_slab


def split_k_plan(plan: "tc.Plan", expr: str, extents: str, world: int, rank: int,
                 index: str | None = None):
    k = index or split_k_index(expr, extents)
    ext = _extents(extents)
    lo, ln = bounds(ext[k], world, rank)
    return (plan.restrict(k, lo, ln) if ln > 0 else None), k, lo, ln


def partial_numel(n: int, world: int) -> int:
    """Elements to allocate for a split-K partial of |C| = n: padded to a multiple of world so
    the reduce-scatter needs no copy (the padding stays zero)."""
    return -(-n // world) * world


def reduce_scatter_sum(partial: torch.Tensor, world: int, rank: int, group=None, n: int | None = None) -> torch.Tensor:
    """Sum the partial C's of all ranks and keep this rank's contiguous part (chunks of
    ceil(n / p)).  `partial` holds n = |C| elements, padded (``partial_numel``) or not.
    NCCL: one reduce-scatter straight from the padded buffer; other backends: all-reduce +
    slice."""
    n = partial.numel() if n is None else n
    chunk = -(-n // world)
    if dist.get_backend(group) == "nccl":
        padded = partial if partial.numel() == chunk * world else torch.cat(
            [partial[:n], partial.new_zeros(chunk * world - n)])   # (unpadded callers only)
        out = partial.new_empty(chunk)
        dist.reduce_scatter_tensor(out, padded, op=dist.ReduceOp.SUM, group=group)
        lo = rank * chunk
        return out[:max(0, min(chunk, n - lo))]
    partial = partial[:n]
    full = partial.clone()
    dist.all_reduce(full, op=dist.ReduceOp.SUM, group=group)
    lo = rank * chunk
    return full[lo:min(n, lo + chunk)]


def execute_split_k(sub, A, B, C_partial, world, rank, alpha=1.0, beta=0.0, execute=None,
                    group=None, n: int | None = None, out_bf16: torch.Tensor | None = None):
    """Each rank: partial C over its k-range (beta applied on rank 0 only; C_partial then holds
    the old C there), then the reduce-scatter.  Returns this rank's chunk of the summed
    result; with `out_bf16` (FP32 partials of a BF16 contraction) the chunk is rounded into
    it once by libtc (tc_round_bf16) and returned."""
    n = C_partial.numel() if n is None else n
    if rank != 0:
        C_partial.zero_()
    b = beta if rank == 0 else 0.0
    if sub is not None:
        (execute or (lambda p, a, bb, c: p.execute(a, bb, c, alpha, b)))(sub, A, B, C_partial[:n])
    elif rank == 0 and beta != 1.0:
        C_partial.mul_(beta)
    part = reduce_scatter_sum(C_partial, world, rank, group, n)
    if out_bf16 is not None:
        tc.round_bf16(out_bf16[:part.numel()], part)
        return out_bf16[:part.numel()]
    return part
