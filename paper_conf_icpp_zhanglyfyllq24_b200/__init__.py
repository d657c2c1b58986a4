"""Python binding of libjigsaw.so (include/jigsaw.h) -- argument marshalling only.

Every step of the hot path (reorder R1..R5, SpMM S1) runs in the CUDA kernels of
``csrc/``; this module only passes pointers, sizes and streams through ctypes.
PyTorch is used for device memory and streams.  There is no CPU fallback: if the
library is missing or the device is not sm_100a, the calls raise.

Names follow the paper's problem statement and the north-star
calls: ``reorder(A, v)`` -> Handle (jigsaw_reorder), ``Handle.spmm(B)``
(jigsaw_spmm), ``Handle.free()`` (jigsaw_free).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libjigsaw.so")

STATUS = {0: "SUCCESS", 1: "INVALID_VALUE", 2: "UNSUPPORTED", 3: "OUT_OF_MEMORY", 4: "CUDA",
          5: "WRONG_DEVICE", 6: "INTERNAL"}

# Every symbol include/jigsaw.h declares (tests check the library exports all of them).
ABI_SYMBOLS = ["jigsaw_reorder", "jigsaw_spmm", "jigsaw_free", "jigsaw_last_status",
               "jigsaw_last_error_string", "jigsaw_version", "jigsaw_reorder_ex",
               "jigsaw_reorder_host", "jigsaw_get_info", "jigsaw_export_format",
               "jigsaw_spmm_host", "jigsaw_spmm_batched", "jigsaw_spmm_batched_host", "jigsaw_spmm_launches_per_call",
               "jigsaw_debug_trace", "jigsaw_last_launch", "jigsaw_set_launch_override", "jigsaw_reorder_batched"]

C_F16, C_F32 = 0, 1            # jigsaw_c_dtype_t
ROWS_GIVEN, ROWS_CLUSTERED = 0, 1   # jigsaw_row_order_t
PANEL_AUTOTUNE = -1                  # panel_rows: time 128- and 256-row formats, keep the faster


class JigsawError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"jigsaw error {STATUS.get(status, status)}: {msg}")
        self.status = status


class Options(ctypes.Structure):
    _fields_ = [("panel_rows", ctypes.c_int), ("residual_mode", ctypes.c_int), ("c_dtype", ctypes.c_int),
                ("row_order", ctypes.c_int), ("autotune_n", ctypes.c_int), ("cc_max_nnz", ctypes.c_int),
                ("reserved", ctypes.c_int * 2)]


class Info(ctypes.Structure):
    _fields_ = [("M", ctypes.c_int64), ("K", ctypes.c_int64), ("v", ctypes.c_int32),
                ("panel_rows", ctypes.c_int32), ("residual_mode", ctypes.c_int32),
                ("device", ctypes.c_int32), ("c_dtype", ctypes.c_int32), ("row_order", ctypes.c_int32),
                ("npanels", ctypes.c_int64), ("ntiles", ctypes.c_int64),
                ("ndtiles", ctypes.c_int64), ("overflow_tiles", ctypes.c_int64),
                ("evictions", ctypes.c_int64), ("nnz", ctypes.c_int64), ("kp_total", ctypes.c_int64),
                ("max_tiles", ctypes.c_int64), ("nksteps", ctypes.c_int64),
                ("format_bytes", ctypes.c_int64), ("device_bytes", ctypes.c_int64),
                ("reorder_ms", ctypes.c_double), ("cc_max_nnz", ctypes.c_int32), ("reserved0", ctypes.c_int32),
                ("cc_tiles", ctypes.c_int64), ("cc_entries", ctypes.c_int64)]


class FormatHost(ctypes.Structure):
    _fields_ = [(n, ctypes.c_void_p) for n in
                ("T", "D", "col_idx", "perm", "gather", "vals", "meta", "kind", "nevict", "rcol", "dvals",
                 "rowmap", "cc_T", "cc_eoff", "cc_row", "cc_col", "cc_val")]


class LaunchDesc(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in
                ("launches", "tile_n", "split_k", "grid", "cta_pair", "problems", "work_items", "split_slots",
                 "dynamic_schedule", "graph_owned_workspace", "nsplit_items")] + [("reserved", ctypes.c_int32 * 5)]


class LaunchOverride(ctypes.Structure):
    _fields_ = [("tile_n", ctypes.c_int32), ("split_k", ctypes.c_int32), ("no_pieces", ctypes.c_int32),
                ("host_chunks", ctypes.c_int32), ("k_pieces", ctypes.c_int32), ("reserved", ctypes.c_int32 * 3)]


_lib = None


def lib(build_if_missing: bool = True):
    """Load libjigsaw.so (building it with nvcc first if it is absent or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    if build_if_missing:
        try:
            _build.build()
        except Exception:
            if not os.path.exists(LIB_PATH):
                raise
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"libjigsaw.so not built ({LIB_PATH}); run __graft_entry__.build()")
    # developer A/B of two builds of the same library (e.g. tools/ab_*.sh)
    L = ctypes.CDLL(os.environ.get("JIGSAW_LIB_AB") or LIB_PATH)
    vp, i64, ci = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
    sig = {
        "jigsaw_reorder": (vp, [vp, i64, i64, ci]),
        "jigsaw_spmm": (ci, [vp, vp, i64, vp, vp]),
        "jigsaw_free": (None, [vp]),
        "jigsaw_last_status": (ci, []),
        "jigsaw_last_error_string": (ctypes.c_char_p, []),
        "jigsaw_version": (ctypes.c_char_p, []),
        "jigsaw_reorder_ex": (ci, [vp, i64, i64, ci, ctypes.POINTER(Options), vp, ctypes.POINTER(vp)]),
        "jigsaw_reorder_host": (ci, [vp, i64, i64, ci, ctypes.POINTER(Options), vp, ctypes.POINTER(vp)]),
        "jigsaw_reorder_batched": (ci, [ctypes.POINTER(vp), ctypes.POINTER(i64), ctypes.POINTER(i64),
                                        ctypes.POINTER(ci), ci, ctypes.POINTER(Options), vp, ctypes.POINTER(vp)]),
        "jigsaw_get_info": (ci, [vp, ctypes.POINTER(Info)]),
        "jigsaw_export_format": (ci, [vp, ctypes.POINTER(FormatHost)]),
        "jigsaw_spmm_host": (ci, [vp, vp, i64, vp, vp]),
        "jigsaw_spmm_batched": (ci, [ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(i64),
                                     ctypes.POINTER(vp), ci, vp]),
        "jigsaw_spmm_batched_host": (ci, [ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(i64),
                                          ctypes.POINTER(vp), ci, vp]),
        "jigsaw_spmm_launches_per_call": (ci, [vp, i64]),
        "jigsaw_debug_trace": (ci, [vp, ci]),
        "jigsaw_last_launch": (ci, [ctypes.POINTER(LaunchDesc)]),
        "jigsaw_set_launch_override": (ci, [ctypes.POINTER(LaunchOverride)]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    _lib = L
    return L


def _raise_if(status: int):
    if status != 0:
        raise JigsawError(status, lib().jigsaw_last_error_string().decode())


def version() -> str:
    return lib().jigsaw_version().decode()


def _stream_ptr(stream):
    if stream is None:
        import torch
        return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return ctypes.c_void_p(stream)
    return ctypes.c_void_p(stream.cuda_stream)


def _check_cuda(t, name, dtype=None):
    import torch
    dtype = dtype or torch.float16
    if not isinstance(t, torch.Tensor) or t.dtype != dtype or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA {dtype} tensor")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous (row-major)")


def _check_fp16_cuda(t, name):
    _check_cuda(t, name)


def _host16(x: np.ndarray, name: str) -> np.ndarray:
    x = np.ascontiguousarray(x)
    if x.dtype == np.float16:
        x = x.view(np.uint16)
    if x.dtype.itemsize != 2 or x.ndim != 2:
        raise TypeError(f"{name} must be a 2-D fp16 (or 16-bit pattern) host array")
    return x


class Handle:
    """A prepared matrix (jigsaw_handle_t): the reorder-aware format on the device."""

    def __init__(self, ptr: int):
        self._h = ctypes.c_void_p(ptr)
        inf = self.info()
        self.M, self.K = inf["M"], inf["K"]
        self.c_dtype = inf["c_dtype"]

    @property
    def c_torch_dtype(self):
        import torch
        return torch.float32 if self.c_dtype == C_F32 else torch.float16

    @property
    def c_numpy_dtype(self):
        return np.float32 if self.c_dtype == C_F32 else np.uint16

    def check_b_c(self, B, C):
        """The checks jigsaw_spmm relies on the caller for: B is a contiguous CUDA
        fp16 K x N tensor, C a contiguous CUDA M x N tensor of the handle's c_dtype."""
        _check_fp16_cuda(B, "B")
        K, N = B.shape
        if K != self.K:
            raise ValueError(f"B has {K} rows, A has K = {self.K}")
        _check_cuda(C, "C", self.c_torch_dtype)
        if tuple(C.shape) != (self.M, N):
            raise ValueError(f"C must be {self.M} x {N}")
        if C.device != B.device:
            raise ValueError("B and C must be on the same device")

    @property
    def ptr(self):
        return self._h

    def info(self) -> dict:
        out = Info()
        _raise_if(lib().jigsaw_get_info(self._h, ctypes.byref(out)))
        return {n: getattr(out, n) for n, _ in Info._fields_}

    def spmm(self, B, C=None, stream=None):
        """C = A x B (jigsaw_spmm); B: CUDA fp16 K x N; returns C (M x N, fp16 or
        fp32 per the handle's c_dtype)."""
        import torch
        _check_fp16_cuda(B, "B")
        N = B.shape[1]
        if C is None:
            C = torch.empty((self.M, N), dtype=self.c_torch_dtype, device=B.device)
        self.check_b_c(B, C)
        _raise_if(lib().jigsaw_spmm(self._h, ctypes.c_void_p(B.data_ptr()), N,
                                    ctypes.c_void_p(C.data_ptr()), _stream_ptr(stream)))
        return C

    def spmm_host(self, B: np.ndarray, out: np.ndarray = None, stream=None) -> np.ndarray:
        """End-to-end path (jigsaw_spmm_host): host B in, host C out (optionally
        into `out`, e.g. pinned memory)."""
        B = _host16(B, "B")
        if B.shape[0] != self.K:
            raise ValueError(f"B has {B.shape[0]} rows, A has K = {self.K}")
        C = np.empty((self.M, B.shape[1]), dtype=self.c_numpy_dtype) if out is None else out
        if (C.shape != (self.M, B.shape[1]) or not C.flags.c_contiguous
                or C.itemsize != np.dtype(self.c_numpy_dtype).itemsize):
            raise ValueError("out must be a contiguous M x N array of the handle's C element size")
        _raise_if(lib().jigsaw_spmm_host(self._h, B.ctypes.data_as(ctypes.c_void_p), B.shape[1],
                                         C.ctypes.data_as(ctypes.c_void_p),
                                         _stream_ptr(stream) if stream is not None else None))
        return C

    def export(self) -> dict:
        """Canonical format (jigsaw_export_format) as numpy arrays."""
        inf = self.info()
        npan, nt, nd, P = inf["npanels"], inf["ntiles"], inf["ndtiles"], inf["panel_rows"]
        ne = inf["cc_entries"]
        arr = dict(T=np.zeros(npan, np.int64), D=np.zeros(npan, np.int64),
                   col_idx=np.zeros((nt, 16), np.int32), perm=np.zeros((nt, 16), np.uint8),
                   gather=np.zeros((nt, 16), np.int32), vals=np.zeros((nt, P, 8), np.uint16),
                   meta=np.zeros((nt, P), np.uint16), kind=np.zeros(nt, np.uint8),
                   nevict=np.zeros(nt, np.uint8), rcol=np.zeros((nd, 16), np.int32),
                   dvals=np.zeros((nd, P, 16), np.uint16), rowmap=np.zeros(inf["M"], np.int32),
                   cc_T=np.zeros(npan, np.int64), cc_eoff=np.zeros(npan + 1, np.int64),
                   cc_row=np.zeros(ne, np.int32), cc_col=np.zeros(ne, np.int32), cc_val=np.zeros(ne, np.uint16))
        fh = FormatHost(**{k: v.ctypes.data for k, v in arr.items()})
        _raise_if(lib().jigsaw_export_format(self._h, ctypes.byref(fh)))
        return arr

    def free(self):
        if self._h is not None and self._h.value:
            lib().jigsaw_free(self._h)
        self._h = ctypes.c_void_p(0)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def reorder(A, v: int, panel_rows: int = 128, residual_mode: int = 0, c_dtype: int = C_F16,
            row_order: int = ROWS_GIVEN, autotune_n: int = 0, cc_max_nnz: int = 0, stream=None) -> Handle:
    """jigsaw_reorder_ex: multi-granularity reorder + format build of A (CUDA fp16 M x K).
    panel_rows = PANEL_AUTOTUNE times both panel heights on an autotune_n-column
    product (0 = 256) and keeps the faster format.  cc_max_nnz = Z > 0 moves the
    tiles with <= Z nonzeros to the CUDA cores (f3, R-Q28)."""
    _check_fp16_cuda(A, "A")
    M, K = A.shape
    opt = Options(panel_rows, residual_mode, c_dtype, row_order, autotune_n, cc_max_nnz)
    out = ctypes.c_void_p(0)
    _raise_if(lib().jigsaw_reorder_ex(ctypes.c_void_p(A.data_ptr()), M, K, v, ctypes.byref(opt),
                                      _stream_ptr(stream), ctypes.byref(out)))
    return Handle(out.value)


def reorder_batched(As, vs, panel_rows: int = 128, residual_mode: int = 0, c_dtype: int = C_F16,
                    row_order: int = ROWS_GIVEN, autotune_n: int = 0, cc_max_nnz: int = 0, stream=None):
    """jigsaw_reorder_batched: the formats of many matrices (CUDA fp16), built
    concurrently on internal streams; returns a list of Handles."""
    n = len(As)
    if len(vs) != n:
        raise ValueError("As and vs must have the same length")
    for A in As:
        _check_fp16_cuda(A, "A")
    opt = Options(panel_rows, residual_mode, c_dtype, row_order, autotune_n, cc_max_nnz)
    ap = (ctypes.c_void_p * n)(*[A.data_ptr() for A in As])
    ms = (ctypes.c_int64 * n)(*[A.shape[0] for A in As])
    ks = (ctypes.c_int64 * n)(*[A.shape[1] for A in As])
    vv = (ctypes.c_int * n)(*vs)
    out = (ctypes.c_void_p * n)()
    _raise_if(lib().jigsaw_reorder_batched(ap, ms, ks, vv, n, ctypes.byref(opt), _stream_ptr(stream), out))
    return [Handle(p) for p in out]


def reorder_host(A: np.ndarray, v: int, panel_rows: int = 128, residual_mode: int = 0,
                 c_dtype: int = C_F16, row_order: int = ROWS_GIVEN, cc_max_nnz: int = 0) -> Handle:
    """jigsaw_reorder_host: A given as a host array (fp16 or uint16 bits)."""
    A = _host16(A, "A")
    M, K = A.shape
    opt = Options(panel_rows, residual_mode, c_dtype, row_order, 0, cc_max_nnz)
    out = ctypes.c_void_p(0)
    _raise_if(lib().jigsaw_reorder_host(A.ctypes.data_as(ctypes.c_void_p), M, K, v,
                                        ctypes.byref(opt), None, ctypes.byref(out)))
    return Handle(out.value)


def debug_trace(max_ctas: int = 1024) -> np.ndarray:
    """Timeline of the last k_spmm launch made with JIGSAW_TRACE=1: [ctas, 24] int64."""
    out = np.zeros((max_ctas, 24), np.int64)
    n = lib().jigsaw_debug_trace(out.ctypes.data_as(ctypes.c_void_p), max_ctas)
    if n < 0:
        raise JigsawError(4, "jigsaw_debug_trace failed")
    return out[:n]


def _addr(x: np.ndarray) -> int:
    """Data address of a host array (cheaper than ``x.ctypes.data``)."""
    return x.__array_interface__["data"][0]


def spmm_batched_host(handles, Bs, outs=None, stream=None):
    """jigsaw_spmm_batched_host: the batch with host B's in and host C's out
    (pinned arrays, e.g. from torch pin_memory, let the copies overlap)."""
    n = len(handles)
    if len(Bs) != n or (outs is not None and len(outs) != n):
        raise ValueError("handles, Bs and outs must have the same length")
    Bs = [_host16(b, "B") for b in Bs]
    if outs is None:
        outs = [np.empty((h.M, b.shape[1]), dtype=h.c_numpy_dtype) for h, b in zip(handles, Bs)]
    for h, b, c in zip(handles, Bs, outs):
        if b.shape[0] != h.K:
            raise ValueError(f"B has {b.shape[0]} rows, A has K = {h.K}")
        if (c.shape != (h.M, b.shape[1]) or not c.flags.c_contiguous
                or c.itemsize != (4 if h.c_dtype == C_F32 else 2)):
            raise ValueError("each out must be a contiguous M x N array of its handle's C element size")
    hs = (ctypes.c_void_p * n)(*[h._h.value for h in handles])
    bp = (ctypes.c_void_p * n)(*[_addr(b) for b in Bs])
    cp = (ctypes.c_void_p * n)(*[_addr(c) for c in outs])
    ns = (ctypes.c_int64 * n)(*[b.shape[1] for b in Bs])
    _raise_if(lib().jigsaw_spmm_batched_host(hs, bp, ns, cp, n, _stream_ptr(stream) if stream is not None else None))
    return outs


def spmm_batched(handles, Bs, Cs, stream=None):
    """jigsaw_spmm_batched: independent products in grouped persistent launches."""
    n = len(handles)
    if len(Bs) != n or len(Cs) != n:
        raise ValueError("handles, Bs and Cs must have the same length")
    for h, b, c in zip(handles, Bs, Cs):
        h.check_b_c(b, c)
    hs = (ctypes.c_void_p * n)(*[h.ptr.value for h in handles])
    bp = (ctypes.c_void_p * n)(*[b.data_ptr() for b in Bs])
    cp = (ctypes.c_void_p * n)(*[c.data_ptr() for c in Cs])
    ns = (ctypes.c_int64 * n)(*[b.shape[1] for b in Bs])
    _raise_if(lib().jigsaw_spmm_batched(hs, bp, ns, cp, n, _stream_ptr(stream)))
    return Cs


def last_launch() -> dict:
    """jigsaw_last_launch: how this thread's most recent SpMM call was launched."""
    d = LaunchDesc()
    _raise_if(lib().jigsaw_last_launch(ctypes.byref(d)))
    return {n: getattr(d, n) for n, _ in LaunchDesc._fields_ if n != "reserved"}


def set_launch_override(tile_n: int = 0, split_k: int = 0, no_pieces: int = 0, host_chunks: int = 0,
                        k_pieces: int = 0):
    """jigsaw_set_launch_override (diagnostic, this thread): force the tile width,
    split-K factor, no splitting / k-range pieces instead of column slices, or the
    host chunk count; all zeros = library choice."""
    o = LaunchOverride(tile_n, split_k, no_pieces, host_chunks, k_pieces)
    _raise_if(lib().jigsaw_set_launch_override(ctypes.byref(o)))


class launch_override:
    """Context manager around set_launch_override (restores the library's choice)."""

    def __init__(self, **kw):
        self.kw = kw

    def __enter__(self):
        set_launch_override(**self.kw)
        return self

    def __exit__(self, *exc):
        set_launch_override()
        return False
