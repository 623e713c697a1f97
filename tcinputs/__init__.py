"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO contraction arithmetic: it only lists the workloads (expression
strings + extents) and draws seeded values.  Both sides (oracle/ and the libtc product)
consume what it returns; neither imports the other.

Workloads:
  * eq. (1) of PAPER.md L43: ``abcd-aebf-dfce``, all extents 16;
  * the TCCG-48 suite (``tccg48.txt``; SURVEY.md Appendix A — reconstructed, since
    PAPER.md lists it only on the Fig. 4/5 axes);
  * CCSD(T) sd_t_d1/d2 6D contractions at uniform extent N.
Values: U(-1, 1) fp64 from ``torch.Generator(device).manual_seed(seed)`` (seeds A=1000+id,
B=2000+id, C_in=3000+id), or integers in [-3, 3] for bitwise-exact runs.  Narrow dtypes
are drawn in fp64 and cast once (RNE).
"""
from __future__ import annotations

import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))

EQ1_EXPR = "abcd-aebf-dfce"
EQ1_EXTENTS = "a:16;b:16;c:16;d:16;e:16;f:16"


@dataclass(frozen=True)
class Case:
    id: int
    expr: str
    extents: str
    conf: str = "-"
    group: str = "-"

    @property
    def ext(self) -> dict:
        return parse_extents(self.extents)


def parse_extents(s: str) -> dict:
    out = {}
    for part in s.split(";"):
        part = part.strip()
        if part:
            k, v = part.split(":")
            out[k.strip()] = int(v)
    return out


def extents_str(d: dict) -> str:
    return ";".join(f"{k}:{v}" for k, v in d.items())


def split_expr(expr: str):
    """'abcd-aebf-dfce' -> ('abcd', 'aebf', 'dfce') — TCCG C-A-B strings only."""
    c, a, b = expr.split("-")
    return c, a, b


def tccg48() -> list[Case]:
    cases = []
    with open(os.path.join(_HERE, "tccg48.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            i, expr, ext, conf, grp = line.split()
            cases.append(Case(int(i), expr, ext, conf, grp))
    assert len(cases) == 48
    return cases


def eq1(n: int = 16) -> Case:
    return Case(0, EQ1_EXPR, ";".join(f"{c}:{n}" for c in "abcdef"), "H", "eq1")


def ccsdt(n: int, expr: str = "abcdef-gdab-efgc", cid: int = 101) -> Case:
    return Case(cid, expr, ";".join(f"{c}:{n}" for c in "abcdefg"), "H", "CCSDT")


def numel(indices: str, ext: dict) -> int:
    n = 1
    for c in indices:
        n *= ext[c]
    return n


def flops(expr: str, extents: str) -> float:
    """2 * prod(all extents) (reading R5; TCCG convention)."""
    ext = parse_extents(extents)
    f = 2.0
    for v in ext.values():
        f *= v
    return f


# ----------------------------------------------------------------- values
def uniform(n: int, seed: int, device="cpu"):
    """U(-1, 1) fp64 torch tensor (flat), from a seeded torch.Generator on `device`."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return torch.rand(n, generator=g, dtype=torch.float64, device=device) * 2 - 1


def integers(n: int, seed: int, lo: int = -3, hi: int = 3, device="cpu"):
    """Integers in [lo, hi] as fp64 (exact in every dtype), seeded."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return torch.randint(lo, hi + 1, (n,), generator=g, device=device).to(torch.float64)


def uniform_np(n: int, seed: int) -> np.ndarray:
    return uniform(n, seed).numpy()


def integers_np(n: int, seed: int, lo: int = -3, hi: int = 3) -> np.ndarray:
    return integers(n, seed, lo, hi).numpy()


def outer_factors(indices: str, ext: dict, seed: int, lo=0.5, hi=1.5):
    """Per-index vectors u_i ~ U(lo, hi) for the rank-1 construction."""
    rng = np.random.default_rng(seed)
    return {c: rng.uniform(lo, hi, ext[c]) for c in indices}


def outer_tensor(indices: str, factors: dict) -> np.ndarray:
    """Flat tensor T[i0, i1, ...] = prod_k factors[idx_k][i_k], first index fastest."""
    t = np.ones(1)
    for c in indices:                      # each new index is slower than all previous
        t = np.multiply.outer(factors[c], t).reshape(-1)
    return t


def bf16_bits(x) -> np.ndarray:
    """fp64 -> bf16 bit patterns (uint16), RNE, via torch's own cast."""
    import torch
    t = torch.as_tensor(np.asarray(x, dtype=np.float64)).to(torch.bfloat16)
    return t.view(torch.int16).numpy().view(np.uint16)


def bf16_to_f64(bits) -> np.ndarray:
    b = np.asarray(bits, dtype=np.uint16).astype(np.uint32) << 16
    return b.view(np.float32).astype(np.float64)
