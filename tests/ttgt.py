"""Independent formulations used to PIN the oracle (tests only; never the product).

* ``ttgt``: the Transpose-Transpose-GEMM-Transpose construction of PAPER.md L50-54
  (Section II): permute A to TA[ext_A..., int...], B to TB[int..., ext_B...], view both
  as matrices MA[i, j], MB[j, k] ("consecutive indexes ... treated as a single virtual
  index"), multiply with a library matmul, and permute MC back to C's order.
* ``einsum_ref``: torch.einsum in fp64 on CPU with every index string reversed (a
  first-index-fastest ``abcd`` tensor is a row-major ``dcba`` array).
Neither shares code with oracle/tc_oracle.c.
"""
from __future__ import annotations

import numpy as np


def _nd(flat, idx, ext):
    """Flat first-index-fastest tensor -> numpy array whose axes are reversed(idx)."""
    return np.asarray(flat).reshape([ext[c] for c in reversed(idx)]) if idx else np.asarray(flat).reshape(())


def ttgt(c_idx: str, a_idx: str, b_idx: str, ext: dict, A, B) -> np.ndarray:
    ext_a = [x for x in a_idx if x in c_idx]
    ext_b = [x for x in b_idx if x in c_idx]
    intl = [x for x in a_idx if x not in c_idx]
    an = _nd(A, a_idx, ext)                      # axes: reversed(a_idx)
    bn = _nd(B, b_idx, ext)
    a_axes = list(reversed(a_idx))
    b_axes = list(reversed(b_idx))
    # TA[ext_a..., int...] and TB[int..., ext_b...] as row-major arrays
    ta = np.transpose(an, [a_axes.index(x) for x in ext_a + intl]) if a_idx else an
    tb = np.transpose(bn, [b_axes.index(x) for x in intl + ext_b]) if b_idx else bn
    m = int(np.prod([ext[x] for x in ext_a])) if ext_a else 1
    k = int(np.prod([ext[x] for x in intl])) if intl else 1
    n = int(np.prod([ext[x] for x in ext_b])) if ext_b else 1
    MA = np.ascontiguousarray(ta).reshape(m, k)   # MA[i, j]
    MB = np.ascontiguousarray(tb).reshape(k, n)   # MB[j, k]
    MC = MA @ MB                                  # GEMM
    tc = MC.reshape([ext[x] for x in ext_a + ext_b])   # TC[ext_a..., ext_b...]
    labels = ext_a + ext_b
    # back to C's storage: row-major axes reversed(c_idx)
    tcn = np.transpose(tc, [labels.index(x) for x in reversed(c_idx)]) if c_idx else tc
    return np.ascontiguousarray(tcn).reshape(-1)


def einsum_ref(c_idx: str, a_idx: str, b_idx: str, ext: dict, A, B) -> np.ndarray:
    import torch
    an = torch.as_tensor(_nd(A, a_idx, ext), dtype=torch.float64)
    bn = torch.as_tensor(_nd(B, b_idx, ext), dtype=torch.float64)
    eq = f"{a_idx[::-1]},{b_idx[::-1]}->{c_idx[::-1]}"
    return torch.einsum(eq, an, bn).reshape(-1).numpy()


def batched_ttgt(c_idx: str, a_idx: str, b_idx: str, ext: dict, A, B) -> np.ndarray:
    """Batch (Hadamard) indices — in C, A and B — by explicit slicing: for every combination
    of the batch indices, take the A, B slices, contract them with ``ttgt`` and write the C
    slice (R31: C[..h..] = sum A[..h..] B[..h..] for each h)."""
    import itertools
    bat = [x for x in c_idx if x in a_idx and x in b_idx]
    if not bat:
        return ttgt(c_idx, a_idx, b_idx, ext, A, B)
    an, bn = _nd(A, a_idx, ext), _nd(B, b_idx, ext)
    cn = np.zeros([ext[x] for x in reversed(c_idx)])
    ra, rb, rc = list(reversed(a_idx)), list(reversed(b_idx)), list(reversed(c_idx))
    for combo in itertools.product(*[range(ext[x]) for x in bat]):
        sel = dict(zip(bat, combo))
        sa = an[tuple(sel.get(x, slice(None)) for x in ra)]
        sb = bn[tuple(sel.get(x, slice(None)) for x in rb)]
        c2, a2, b2 = ("".join(x for x in s if x not in bat) for s in (c_idx, a_idx, b_idx))
        flat = ttgt(c2, a2, b2, ext, np.ascontiguousarray(sa).reshape(-1), np.ascontiguousarray(sb).reshape(-1))
        cn[tuple(sel.get(x, slice(None)) for x in rc)] = _nd(flat, c2, ext)
    return cn.reshape(-1)
