"""CPU oracle for direct tensor contraction — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product (``libtc``) never
imports it and shares no code with it.

What it computes (Section II, eq. (1)): ``C = alpha * sum_int A*B +
beta * C`` with the Einstein convention, each index in exactly two tensors
(P:L64), first listed index stride-1.  The C library
``libtc_oracle.so`` (``oracle/tc_oracle.c``) is the plain nested loop of P:L62; this
module is argument marshalling (numpy <-> ctypes) only.

Parity status: pinned — see tests/test_oracle.py (TTGT brute force per P:L50-54, GEMM
special cases, rank-1 closed form, constant / delta inputs, linearity, relabelling,
operand swap, output permutation, slab consistency, Neumaier self-check).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "tc_oracle.c")
# gcc flags of SURVEY 8(d) / BASELINE.md: the plain loop at -O3 for this host's own ISA;
# -ffp-contract=off so each term is a plain multiply followed by a plain add
CFLAGS = ["-O3", "-march=native", "-fopenmp", "-ffp-contract=off", "-fPIC", "-shared"]


def cpu_model() -> str:
    """The host CPU's model name (/proc/cpuinfo), for the bench line."""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def _host_key() -> str:
    # -march=native code is only valid on the CPU it was compiled for: one library per host
    # ISA (the tree travels to the GPU box, where the oracle is rebuilt for that host)
    import hashlib
    flags = ""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("flags"):
                    flags = line
                    break
    except OSError:
        pass
    return hashlib.sha1((cpu_model() + flags).encode()).hexdigest()[:12]


_SO = os.path.join(_HERE, f"libtc_oracle_{_host_key()}.so")

STATUS = {0: "TC_SUCCESS", 1: "TC_ERR_INVALID_ARG", 2: "TC_ERR_PARSE", 3: "TC_ERR_INDEX",
          4: "TC_ERR_EXTENT", 5: "TC_ERR_UNSUPPORTED"}
DTYPES = {"f64": 0, "f32": 1, "tf32": 2, "bf16": 3}
_NP = {"f64": np.float64, "f32": np.float32, "tf32": np.float32, "bf16": np.uint16}


def build(force: bool = False) -> str:
    """Compile the oracle (plain C, -O3 -march=native, -ffp-contract=off so each term is
    mul-then-add) for this host."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = f"{_SO}.{os.getpid()}.tmp"
        subprocess.check_call(["gcc"] + CFLAGS + ["-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _SO)
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        c, vp, dp, i64 = ctypes.c_char_p, ctypes.c_void_p, ctypes.c_double, ctypes.c_int64
        L.tco_check.argtypes = [c, c]
        L.tco_check.restype = ctypes.c_int
        L.tco_numel.argtypes = [c, c, ctypes.c_int]
        L.tco_numel.restype = i64
        L.tco_range.argtypes = [c, c, ctypes.c_int, vp, vp, vp, vp, vp, dp, dp, i64, i64,
                                ctypes.c_int, ctypes.c_int]
        L.tco_range.restype = ctypes.c_int
        L.tco_sample.argtypes = [c, c, ctypes.c_int, vp, vp, vp, vp, vp, dp, dp, vp, i64,
                                 ctypes.c_int, ctypes.c_int]
        L.tco_sample.restype = ctypes.c_int
        L.tco_max_threads.restype = ctypes.c_int
        _lib = L
    return _lib


class OracleError(RuntimeError):
    def __init__(self, status: int):
        super().__init__(STATUS.get(status, str(status)))
        self.status = status


def check(expr: str, extents: str) -> str:
    """Parse + validate; returns the status name (same names as libtc's tc_status_t)."""
    return STATUS[lib().tco_check(expr.encode(), extents.encode())]


def numel(expr: str, extents: str, which: str) -> int:
    n = lib().tco_numel(expr.encode(), extents.encode(), "CAB".index(which))
    if n < 0:
        raise OracleError(lib().tco_check(expr.encode(), extents.encode()))
    return int(n)


def _ptr(a):
    return None if a is None else a.ctypes.data


def _prep(a, dtype):
    return None if a is None else np.ascontiguousarray(a, dtype=_NP[dtype]).reshape(-1)


def contract(expr, extents, A, B, C=None, alpha=1.0, beta=0.0, dtype="f64", lo=0, hi=None,
             exact=False, with_scale=False, nthreads=0):
    """C linear indices [lo, hi) of alpha*sum A*B + beta*C (flat, first index fastest)."""
    A, B, C = _prep(A, dtype), _prep(B, dtype), _prep(C, dtype)
    if hi is None:
        hi = numel(expr, extents, "C")
    out = np.empty(hi - lo, dtype=_NP[dtype])
    S = np.empty(hi - lo, dtype=np.float64) if with_scale else None
    st = lib().tco_range(expr.encode(), extents.encode(), DTYPES[dtype], _ptr(A), _ptr(B), _ptr(C),
                         _ptr(out), _ptr(S), float(alpha), float(beta), int(lo), int(hi),
                         int(exact), int(nthreads))
    if st:
        raise OracleError(st)
    return (out, S) if with_scale else out


def sample(expr, extents, A, B, idx, C=None, alpha=1.0, beta=0.0, dtype="f64", exact=False,
           with_scale=False, nthreads=0):
    """The C elements at the given linear indices."""
    A, B, C = _prep(A, dtype), _prep(B, dtype), _prep(C, dtype)
    idx = np.ascontiguousarray(idx, dtype=np.int64).reshape(-1)
    out = np.empty(idx.size, dtype=_NP[dtype])
    S = np.empty(idx.size, dtype=np.float64) if with_scale else None
    st = lib().tco_sample(expr.encode(), extents.encode(), DTYPES[dtype], _ptr(A), _ptr(B),
                          _ptr(C), _ptr(out), _ptr(S), float(alpha), float(beta), _ptr(idx),
                          int(idx.size), int(exact), int(nthreads))
    if st:
        raise OracleError(st)
    return (out, S) if with_scale else out


def max_threads() -> int:
    return int(lib().tco_max_threads())
