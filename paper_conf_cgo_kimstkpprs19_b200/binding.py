"""Thin ctypes binding of libtc (include/libtc.h) — argument marshalling only.

Every step of the contraction runs in libtc.so's CUDA kernels; this module never computes
anything itself and never falls back to another implementation: if libtc.so is missing or a
call fails, it raises.  torch is used for device memory and streams only.

Layout: the FIRST listed index of each tensor is stride-1, so a torch
tensor for index list "aebf" has shape (N_f, N_b, N_e, N_a) (reversed) and is contiguous;
``empty(plan, "A")`` allocates it.
"""
from __future__ import annotations

import ctypes
import json
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.environ.get("LIBTC_SO") or os.path.join(_HERE, "libtc.so")   # (A/B builds)

STATUS = ["TC_SUCCESS", "TC_ERR_INVALID_ARG", "TC_ERR_PARSE", "TC_ERR_INDEX", "TC_ERR_EXTENT",
          "TC_ERR_UNSUPPORTED", "TC_ERR_NO_CONFIG", "TC_ERR_CUDA", "TC_ERR_ALLOC"]
DTYPES = {"f64": 0, "f32": 1, "tf32": 2, "bf16": 3}
# torch storage dtype per plan dtype (tf32 and f32 both store FP32)
def _tdt(name):
    def get():
        import torch
        return getattr(torch, name)
    return get


_TORCH_DTYPE = {"f64": _tdt("float64"), "f32": _tdt("float32"), "tf32": _tdt("float32"),
                "bf16": _tdt("bfloat16")}
COST = {"b200": 0, "paper": 1}
SLAB_A, SLAB_B, SLAB_C = 1, 2, 4


class TcError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{STATUS[status] if 0 <= status < len(STATUS) else status}: {detail}")
        self.status = STATUS[status] if 0 <= status < len(STATUS) else str(status)
        self.detail = detail


class _Opts(ctypes.Structure):
    _fields_ = [("cost_mode", ctypes.c_int), ("host_only", ctypes.c_int), ("variant", ctypes.c_int),
                ("force_tiles", ctypes.c_char_p), ("no_fusion", ctypes.c_int), ("tma_epilogue", ctypes.c_int),
                ("morder", ctypes.c_int), ("no_tma_operands", ctypes.c_int),
                ("cta_pair", ctypes.c_int), ("out_f32", ctypes.c_int), ("stream", ctypes.c_int),
                ("stream_rank", ctypes.c_int), ("reserved", ctypes.c_int * 1)]


_lib = None


def lib():
    """Load libtc.so (built in-tree by build.py / __graft_entry__.build())."""
    global _lib
    if _lib is None:
        if not os.path.exists(_SO):
            raise ImportError(f"libtc.so not built ({_SO}); run __graft_entry__.build()")
        L = ctypes.CDLL(_SO)
        vp, cp, i64, dbl = ctypes.c_void_p, ctypes.c_char_p, ctypes.c_int64, ctypes.c_double
        L.tc_plan_ex.argtypes = [ctypes.POINTER(vp), cp, cp, ctypes.c_int, ctypes.POINTER(_Opts)]
        L.tc_plan_ex.restype = ctypes.c_int
        L.tc_plan.argtypes = [ctypes.POINTER(vp), cp, cp, ctypes.c_int]
        L.tc_plan.restype = ctypes.c_int
        L.tc_execute.argtypes = [vp, vp, vp, vp, dbl, dbl, vp]
        L.tc_execute.restype = ctypes.c_int
        L.tc_execute_group.argtypes = [ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(vp),
                                       ctypes.c_int, vp, dbl, dbl, vp]
        L.tc_execute_group.restype = ctypes.c_int
        L.tc_execute_host.argtypes = [vp, vp, vp, vp, dbl, dbl, vp, ctypes.c_size_t, vp]
        L.tc_execute_host.restype = ctypes.c_int
        L.tc_plan_workspace_bytes.argtypes = [vp]
        L.tc_plan_workspace_bytes.restype = ctypes.c_size_t
        L.tc_plan_restrict.argtypes = [ctypes.POINTER(vp), vp, cp, i64, i64, ctypes.c_uint]
        L.tc_plan_restrict.restype = ctypes.c_int
        L.tc_plan_tuned.argtypes = [ctypes.POINTER(vp), vp, vp, vp, vp, ctypes.c_int, ctypes.c_int, vp]
        L.tc_plan_tuned.restype = ctypes.c_int
        L.tc_plan_tuned_beta.argtypes = [ctypes.POINTER(vp), vp, vp, vp, vp, ctypes.c_int, ctypes.c_int, dbl, vp]
        L.tc_plan_tuned_beta.restype = ctypes.c_int
        L.tc_plan_info.argtypes = [vp, ctypes.c_char_p, ctypes.c_size_t, ctypes.POINTER(ctypes.c_size_t)]
        L.tc_plan_info.restype = ctypes.c_int
        L.tc_plan_flops.argtypes = [vp]
        L.tc_plan_flops.restype = dbl
        L.tc_plan_numel.argtypes = [vp, ctypes.c_int]
        L.tc_plan_numel.restype = i64
        L.tc_plan_resize.argtypes = [ctypes.POINTER(vp), vp, cp]
        L.tc_plan_resize.restype = ctypes.c_int
        L.tc_plan_select.argtypes = [ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.c_int, cp, ctypes.POINTER(ctypes.c_int)]
        L.tc_plan_select.restype = ctypes.c_int
        L.tc_round_bf16.argtypes = [vp, vp, i64, vp]
        L.tc_round_bf16.restype = ctypes.c_int
        L.tc_plan_span.argtypes = [vp, ctypes.c_int]
        L.tc_plan_span.restype = i64
        p64 = ctypes.POINTER(i64)
        L.tc_plan_strided.argtypes = [ctypes.POINTER(vp), cp, cp, ctypes.c_int, p64, p64, p64, ctypes.POINTER(_Opts)]
        L.tc_plan_strided.restype = ctypes.c_int
        L.tc_plan_destroy.argtypes = [vp]
        L.tc_plan_destroy.restype = None
        L.tc_status_string.argtypes = [ctypes.c_int]
        L.tc_status_string.restype = cp
        L.tc_last_error.restype = cp
        L.tc_version.restype = cp
        L.tc_plan_cached.argtypes = [ctypes.POINTER(vp), cp, cp, ctypes.c_int, ctypes.POINTER(_Opts)]
        L.tc_plan_cached.restype = ctypes.c_int
        L.tc_plan_cache_size.restype = ctypes.c_size_t
        L.tc_plan_cache_clear.restype = None
        L.tc_group_plan.argtypes = [ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.c_int]
        L.tc_group_plan.restype = ctypes.c_int
        L.tc_group_execute.argtypes = [vp, ctypes.POINTER(vp), ctypes.POINTER(vp), vp, dbl, dbl, vp]
        L.tc_group_execute.restype = ctypes.c_int
        L.tc_group_info.argtypes = [vp, ctypes.c_char_p, ctypes.c_size_t, ctypes.POINTER(ctypes.c_size_t)]
        L.tc_group_info.restype = ctypes.c_int
        L.tc_group_destroy.argtypes = [vp]
        L.tc_group_destroy.restype = None
        L.tc_check.argtypes = [cp, cp]
        L.tc_check.restype = ctypes.c_int
        _lib = L
    return _lib


def _raise(st: int):
    if st != 0:
        raise TcError(st, lib().tc_last_error().decode())


def check(expr: str, extents: str) -> str:
    """Parse + validate only; returns the status name."""
    return STATUS[lib().tc_check(expr.encode(), extents.encode())]


def version() -> str:
    return lib().tc_version().decode()


def _stream_ptr(stream):
    if stream is None:
        import torch
        if torch.cuda.is_available():
            return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
        return ctypes.c_void_p(0)
    if isinstance(stream, int):
        return ctypes.c_void_p(stream)
    return ctypes.c_void_p(stream.cuda_stream)


class Plan:
    """A libtc plan (tc_plan_t).  Immutable; execute() may be called any number of times."""

    def __init__(self, handle: ctypes.c_void_p, expr: str, extents: str, dtype: str):
        self._h = handle
        self.expr, self.extents, self.dtype = expr, extents, dtype
        self._info = None

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _lib is not None:
            _lib.tc_plan_destroy(h)
            self._h = None

    @property
    def handle(self):
        return self._h

    def info(self) -> dict:
        if self._info is None:
            need = ctypes.c_size_t(0)
            _raise(lib().tc_plan_info(self._h, None, 0, ctypes.byref(need)))
            buf = ctypes.create_string_buffer(need.value)
            _raise(lib().tc_plan_info(self._h, buf, need.value, ctypes.byref(need)))
            self._info = json.loads(buf.value.decode())
        return self._info

    @property
    def flops(self) -> float:
        return lib().tc_plan_flops(self._h)

    def numel(self, which: str) -> int:
        return int(lib().tc_plan_numel(self._h, "CAB".index(which)))

    def resize(self, extents: str) -> "Plan":
        """tc_plan_resize: this plan's configuration bound to other extents (NEXT-1)."""
        h = ctypes.c_void_p()
        _raise(lib().tc_plan_resize(ctypes.byref(h), self._h, extents.encode()))
        return Plan(h, self.expr, extents, self.dtype)

    def span(self, which: str) -> int:
        """Elements tensor `which`'s buffer must hold (largest offset + 1)."""
        return int(lib().tc_plan_span(self._h, "CAB".index(which)))

    def workspace_bytes(self) -> int:
        return int(lib().tc_plan_workspace_bytes(self._h))

    def restrict(self, index: str, begin: int, length: int, flags: int = 0) -> "Plan":
        h = ctypes.c_void_p()
        _raise(lib().tc_plan_restrict(ctypes.byref(h), self._h, index.encode(), int(begin),
                                      int(length), int(flags)))
        return Plan(h, self.expr, f"{self.extents}|{index}[{begin}:{begin + length}]", self.dtype)

    def tuned(self, A, B, C, topk: int = 4, reps: int = 3, stream=None, beta: float = 0.0) -> "Plan":
        """tc_plan_tuned: time the best configs of the top-k variants on these tensors (C is
        overwritten; with beta != 0, tc_plan_tuned_beta: C is accumulated into) and return
        the fastest as a new plan."""
        for name, t in (("A", A), ("B", B), ("C", C)):
            if not t.is_cuda or not t.is_contiguous():
                raise TcError(1, f"{name} must be a contiguous CUDA tensor")
        h = ctypes.c_void_p()
        _raise(lib().tc_plan_tuned_beta(ctypes.byref(h), self._h, ctypes.c_void_p(A.data_ptr()),
                                        ctypes.c_void_p(B.data_ptr()), ctypes.c_void_p(C.data_ptr()),
                                        int(topk), int(reps), float(beta), _stream_ptr(stream)))
        return Plan(h, self.expr, self.extents, self.dtype)

    def execute_ptr(self, A: int, B: int, C: int, alpha=1.0, beta=0.0, stream=None):
        _raise(lib().tc_execute(self._h, ctypes.c_void_p(A), ctypes.c_void_p(B), ctypes.c_void_p(C),
                                float(alpha), float(beta), _stream_ptr(stream)))

    def execute(self, A, B, C, alpha=1.0, beta=0.0, stream=None):
        """C = alpha * sum A*B + beta * C on torch CUDA tensors (current stream)."""
        want = _TORCH_DTYPE[self.dtype]()
        import torch
        for name, t, w in (("A", A, "A"), ("B", B, "B"), ("C", C, "C")):
            if w == "C" and self.dtype == "bf16" and self.info().get("out_f32"):
                want = torch.float32
            if not t.is_cuda or not t.is_contiguous():
                raise TcError(1, f"{name} must be a contiguous CUDA tensor")
            if t.dtype != want:
                raise TcError(1, f"{name} is {t.dtype}, the plan's dtype {self.dtype!r} needs {want}")
            if t.numel() < self.span(w):
                raise TcError(1, f"{name} holds {t.numel()} elements, the plan's view spans {self.span(w)}")
        self.execute_ptr(A.data_ptr(), B.data_ptr(), C.data_ptr(), alpha, beta, stream)
        return C

    def execute_host(self, A, B, C, workspace, alpha=1.0, beta=0.0, stream=None):
        """End-to-end: host (pinned) A, B, C; device workspace of workspace_bytes()."""
        _raise(lib().tc_execute_host(self._h, ctypes.c_void_p(A.data_ptr()), ctypes.c_void_p(B.data_ptr()),
                                     ctypes.c_void_p(C.data_ptr()), float(alpha), float(beta),
                                     ctypes.c_void_p(workspace.data_ptr()),
                                     ctypes.c_size_t(workspace.numel() * workspace.element_size()),
                                     _stream_ptr(stream)))
        return C


def _opts(cost, host_only, variant, force_tiles, fusion, tma, morder, tma_operands=True, pair=None,
          out_f32=False, stream=None, stream_rank=0) -> _Opts:
    o = _Opts()
    o.stream = {None: 0, False: 1, True: 2}[stream]
    o.stream_rank = int(stream_rank)
    o.out_f32 = int(out_f32)
    o.no_tma_operands = int(not tma_operands)
    o.cta_pair = {None: 0, False: 1, True: 2}[pair]
    o.morder = {None: 0, "C": 1, "X": 2}[morder]
    o.tma_epilogue = int(tma)
    o.cost_mode = COST[cost]
    o.host_only = int(host_only)
    o.variant = 0 if variant is None else int(variant) + 1
    o.force_tiles = force_tiles.encode() if force_tiles else None
    o.no_fusion = int(not fusion)
    return o


def plan_cached(expr: str, extents: str, dtype: str = "f64", cost: str = "b200", host_only: bool = False,
                variant: int | None = None, force_tiles: str | None = None, fusion: bool = True,
                tma: bool = False, morder: str | None = None, tma_operands: bool = True,
                pair: bool | None = None) -> Plan:
    """tc_plan_cached: the process-wide cached plan of these arguments (planned on first use)."""
    o = _opts(cost, host_only, variant, force_tiles, fusion, tma, morder, tma_operands, pair)
    h = ctypes.c_void_p()
    _raise(lib().tc_plan_cached(ctypes.byref(h), expr.encode(), extents.encode(), DTYPES[dtype], ctypes.byref(o)))
    p = Plan(h, expr, extents, dtype)
    p._opts = o
    return p


def execute_group_ptr(plans, A, B, C: int, alpha=1.0, beta=0.0, stream=None):
    """tc_execute_group on raw device pointers: C = alpha * sum_i plans[i](A[i], B[i]) + beta * C."""
    n = len(plans)
    if len(A) != n or len(B) != n:
        raise TcError(1, "plans, A and B must have the same length")
    arr = ctypes.c_void_p * max(n, 1)
    _raise(lib().tc_execute_group(arr(*[p._h for p in plans]), arr(*[ctypes.c_void_p(a) for a in A]),
                                  arr(*[ctypes.c_void_p(b) for b in B]), int(n), ctypes.c_void_p(C),
                                  float(alpha), float(beta), _stream_ptr(stream)))


def execute_group(plans, A, B, C, alpha=1.0, beta=0.0, stream=None):
    """Grouped contractions into one C (CCSD(T) triples pattern) on torch
    CUDA tensors: C = alpha * sum_i plans[i](A[i], B[i]) + beta * C."""
    for name, t in [("C", C)] + [(f"A[{i}]", a) for i, a in enumerate(A)] + [(f"B[{i}]", b) for i, b in enumerate(B)]:
        if not t.is_cuda or not t.is_contiguous():
            raise TcError(1, f"{name} must be a contiguous CUDA tensor")
    execute_group_ptr(plans, [a.data_ptr() for a in A], [b.data_ptr() for b in B], C.data_ptr(),
                      alpha, beta, stream)
    return C


class GroupPlan:
    """A fused grouped contraction (tc_group_t): one kernel computes
    C = alpha * sum_i plans[i](A[i], B[i]) + beta * C with every C tile kept on chip across the
    members and stored once."""

    def __init__(self, handle: ctypes.c_void_p, n: int):
        self._h = handle
        self.n = n
        self._info = None

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _lib is not None:
            _lib.tc_group_destroy(h)
            self._h = None

    def info(self) -> dict:
        if self._info is None:
            need = ctypes.c_size_t(0)
            _raise(lib().tc_group_info(self._h, None, 0, ctypes.byref(need)))
            buf = ctypes.create_string_buffer(need.value)
            _raise(lib().tc_group_info(self._h, buf, need.value, ctypes.byref(need)))
            self._info = json.loads(buf.value.decode())
        return self._info

    def execute_ptr(self, A, B, C: int, alpha=1.0, beta=0.0, stream=None):
        if len(A) != self.n or len(B) != self.n:
            raise TcError(1, f"the group has {self.n} members")
        arr = ctypes.c_void_p * self.n
        _raise(lib().tc_group_execute(self._h, arr(*[ctypes.c_void_p(a) for a in A]),
                                      arr(*[ctypes.c_void_p(b) for b in B]), ctypes.c_void_p(C),
                                      float(alpha), float(beta), _stream_ptr(stream)))

    def execute(self, A, B, C, alpha=1.0, beta=0.0, stream=None):
        import torch
        for name, t in [("C", C)] + [(f"A[{i}]", a) for i, a in enumerate(A)] + [(f"B[{i}]", b) for i, b in enumerate(B)]:
            if not t.is_cuda or not t.is_contiguous():
                raise TcError(1, f"{name} must be a contiguous CUDA tensor")
            if t.dtype != torch.float64:
                raise TcError(1, f"{name} is {t.dtype}; fused groups are FP64")
        self.execute_ptr([a.data_ptr() for a in A], [b.data_ptr() for b in B], C.data_ptr(), alpha, beta, stream)
        return C


def plan_group(plans) -> GroupPlan:
    """tc_group_plan: fuse the member plans (all giving C one layout) into one kernel."""
    n = len(plans)
    arr = ctypes.c_void_p * max(n, 1)
    h = ctypes.c_void_p()
    _raise(lib().tc_group_plan(ctypes.byref(h), arr(*[p._h for p in plans]), int(n)))
    return GroupPlan(h, n)


def plan_cache_size() -> int:
    return int(lib().tc_plan_cache_size())


def plan_cache_clear() -> None:
    lib().tc_plan_cache_clear()


def plan(expr: str, extents: str, dtype: str = "f64", cost: str = "b200", host_only: bool = False,
         variant: int | None = None, force_tiles: str | None = None, fusion: bool = True,
         tma: bool = False, morder: str | None = None, tma_operands: bool = True,
         pair: bool | None = None, out_f32: bool = False, stream: bool | None = None,
         stream_rank: int = 0) -> Plan:
    """pair: None = planner's choice, False / True = CTA pairs off / on where the plan allows.
    stream: None = planner's choice, False / True = the streaming path (bf16 tensor x matrix) off /
    on where eligible.
    out_f32 (bf16 plans): C is FP32 (split-K partials).
    morder: None = planner's choice, "C" = m digits in C order, "X" = in the X operand's order."""
    o = _opts(cost, host_only, variant, force_tiles, fusion, tma, morder, tma_operands, pair, out_f32, stream,
              stream_rank)
    h = ctypes.c_void_p()
    _raise(lib().tc_plan_ex(ctypes.byref(h), expr.encode(), extents.encode(), DTYPES[dtype], ctypes.byref(o)))
    p = Plan(h, expr, extents, dtype)
    p._opts = o  # keep force_tiles bytes alive for the call's duration
    return p


def plan_strided(expr: str, extents: str, strides: dict, dtype: str = "f64", cost: str = "b200",
                 host_only: bool = False, variant: int | None = None, force_tiles: str | None = None,
                 fusion: bool = True) -> Plan:
    """tc_plan_strided: strides = {"C": [...], "A": [...], "B": [...]} (element strides per index
    in the expression's letter order; a missing tensor is dense)."""
    o = _opts(cost, host_only, variant, force_tiles, fusion, False, None)
    arrs = []
    for t in "CAB":
        s = strides.get(t)
        arrs.append(None if s is None else (ctypes.c_int64 * len(s))(*[int(x) for x in s]))
    h = ctypes.c_void_p()
    _raise(lib().tc_plan_strided(ctypes.byref(h), expr.encode(), extents.encode(), DTYPES[dtype],
                                 *[None if a is None else ctypes.cast(a, ctypes.POINTER(ctypes.c_int64)) for a in arrs],
                                 ctypes.byref(o)))
    p = Plan(h, expr, extents, dtype)
    p._opts = o
    return p


def round_bf16(dst, src, stream=None):
    """tc_round_bf16: dst (torch bfloat16, CUDA) = src (float32) rounded RNE, by libtc."""
    import torch
    if dst.dtype != torch.bfloat16 or src.dtype != torch.float32 or dst.numel() < src.numel():
        raise TcError(1, "round_bf16 wants a bfloat16 dst at least as long as the float32 src")
    if not (dst.is_cuda and src.is_cuda and dst.is_contiguous() and src.is_contiguous()):
        raise TcError(1, "round_bf16 wants contiguous CUDA tensors")
    _raise(lib().tc_round_bf16(ctypes.c_void_p(dst.data_ptr()), ctypes.c_void_p(src.data_ptr()),
                               src.numel(), _stream_ptr(stream)))
    return dst


def select(versions, extents: str):
    """tc_plan_select: (plan at `extents`, index of the version the cost model chose)."""
    arr = (ctypes.c_void_p * len(versions))(*[v._h for v in versions])
    h, ch = ctypes.c_void_p(), ctypes.c_int(-1)
    _raise(lib().tc_plan_select(ctypes.byref(h), arr, len(versions), extents.encode(), ctypes.byref(ch)))
    return Plan(h, versions[0].expr, extents, versions[0].dtype), ch.value


def shape_of(indices: str, extents: dict) -> tuple:
    """torch shape of a tensor with the given index list (reversed: first index fastest)."""
    return tuple(extents[c] for c in reversed(indices))
