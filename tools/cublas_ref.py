"""cuBLAS dense fp16 GEMM baselines for bench.py (SURVEY §8(d) "cuBLAS baseline";
PAPER.md P:242 cublasHgemm).  Library code on the BASELINE side only: the
Jigsaw path never calls it.

ctypes binding of the cuBLAS v2 API that torch already loaded (same process,
same library build as torch.matmul):
  * gemm(A, B, C, compute)          -- cublasGemmEx, one row-major product
  * gemm_strided_batched(...)       -- cublasGemmStridedBatchedEx, a stack of
                                       same-shape products in one call
with compute = "16F" (CUBLAS_COMPUTE_16F, the paper's HGemm: fp16 accumulate)
or "32F" (CUBLAS_COMPUTE_32F: fp32 accumulate, fp16 out).  Row-major C = A.B
is issued as the column-major C^T = B^T.A^T (no copies).
"""
from __future__ import annotations

import ctypes
import glob
import os

import numpy as np

CUDA_R_16F = 2
COMPUTE = {"16F": 64, "32F": 68}      # cublasComputeType_t
CUBLAS_OP_N = 0
CUBLAS_GEMM_DEFAULT = -1

_lib = None
_handles = {}


def _load():
    global _lib
    if _lib is not None:
        return _lib
    import torch  # noqa: F401 -- loads the bundled cuBLAS first
    cands = []
    try:
        import nvidia.cublas
        for p in nvidia.cublas.__path__:
            cands += glob.glob(os.path.join(p, "lib", "libcublas.so*"))
    except Exception:
        pass
    cands += ["libcublas.so.12", "libcublas.so"]
    last = None
    for c in cands:
        try:
            L = ctypes.CDLL(c)
            break
        except OSError as e:
            last = e
    else:
        raise OSError(f"libcublas not found: {last}")
    vp, ci, i64 = ctypes.c_void_p, ctypes.c_int, ctypes.c_longlong
    L.cublasCreate_v2.argtypes = [ctypes.POINTER(vp)]
    L.cublasCreate_v2.restype = ci
    L.cublasSetStream_v2.argtypes = [vp, vp]
    L.cublasSetStream_v2.restype = ci
    L.cublasGemmEx.argtypes = [vp, ci, ci, ci, ci, ci, vp, vp, ci, ci, vp, ci, ci, vp, vp, ci, ci, ci, ci]
    L.cublasGemmEx.restype = ci
    L.cublasGemmStridedBatchedEx.argtypes = [vp, ci, ci, ci, ci, ci, vp, vp, ci, ci, i64, vp, ci, ci, i64,
                                             vp, vp, ci, ci, i64, ci, ci, ci]
    L.cublasGemmStridedBatchedEx.restype = ci
    _lib = L
    return L


def _handle(stream_ptr: int):
    L = _load()
    import torch
    dev = torch.cuda.current_device()
    h = _handles.get(dev)
    if h is None:
        h = ctypes.c_void_p()
        st = L.cublasCreate_v2(ctypes.byref(h))
        if st:
            raise RuntimeError(f"cublasCreate failed ({st})")
        _handles[dev] = h
    st = L.cublasSetStream_v2(h, ctypes.c_void_p(stream_ptr))
    if st:
        raise RuntimeError(f"cublasSetStream failed ({st})")
    return h


def _scalars(compute: str):
    if compute == "16F":
        one = np.array([1.0], np.float16)
        zero = np.array([0.0], np.float16)
    else:
        one = np.array([1.0], np.float32)
        zero = np.array([0.0], np.float32)
    return one, zero


def gemm(A, B, C, compute: str = "32F"):
    """C (M x N) = A (M x K) . B (K x N), row-major fp16 CUDA tensors."""
    import torch
    M, K = A.shape
    N = B.shape[1]
    h = _handle(torch.cuda.current_stream().cuda_stream)
    one, zero = _scalars(compute)
    st = _load().cublasGemmEx(h, CUBLAS_OP_N, CUBLAS_OP_N, N, M, K, one.ctypes.data,
                              B.data_ptr(), CUDA_R_16F, N, A.data_ptr(), CUDA_R_16F, K,
                              zero.ctypes.data, C.data_ptr(), CUDA_R_16F, N,
                              COMPUTE[compute], CUBLAS_GEMM_DEFAULT)
    if st:
        raise RuntimeError(f"cublasGemmEx failed ({st})")
    return C


def gemm_strided_batched(A, B, C, compute: str = "32F"):
    """C[i] = A[i] . B[i] for stacked row-major fp16 tensors [b, M, K] x [b, K, N]."""
    import torch
    b, M, K = A.shape
    N = B.shape[2]
    h = _handle(torch.cuda.current_stream().cuda_stream)
    one, zero = _scalars(compute)
    st = _load().cublasGemmStridedBatchedEx(h, CUBLAS_OP_N, CUBLAS_OP_N, N, M, K, one.ctypes.data,
                                            B.data_ptr(), CUDA_R_16F, N, K * N,
                                            A.data_ptr(), CUDA_R_16F, K, M * K,
                                            zero.ctypes.data, C.data_ptr(), CUDA_R_16F, N, M * N,
                                            b, COMPUTE[compute], CUBLAS_GEMM_DEFAULT)
    if st:
        raise RuntimeError(f"cublasGemmStridedBatchedEx failed ({st})")
    return C
