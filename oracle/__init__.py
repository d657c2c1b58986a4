"""CPU oracle for the Jigsaw hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` leg may import this package.  The product path
(``paper_conf_icpp_zhanglyfyllq24_b200``) never imports it, and this package
never imports the product: the two share no code.  The only module both use is
``synth`` (seeded input generators, none of the method's arithmetic).

Thin ctypes marshalling around ``oracle/oracle.c`` (O1 SpMM, O2 canonical
reorder CR1) plus re-exports of the independent numpy checker ``check.py`` (O3).
Citations are to /root/reference/PAPER.md lines (P:NNN) and to the readings
R-Qn listed in DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

PAD = -1


def build(force: bool = False) -> str:
    """Compile oracle.c into liboracle.so with gcc (plain C11, -O2, no SIMD flags)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-shared", "-fPIC",
                               "-o", _LIB, _SRC])
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        i64, p = ctypes.c_int64, ctypes.c_void_p
        L.orc_half_to_double.restype = ctypes.c_double
        L.orc_half_to_double.argtypes = [ctypes.c_uint16]
        L.orc_spmm.restype = ctypes.c_int
        L.orc_spmm.argtypes = [p, i64, i64, p, i64, p, i64, p, p]
        L.orc_tile_reorder.restype = ctypes.c_int
        L.orc_tile_reorder.argtypes = [p, ctypes.c_int, ctypes.c_int, ctypes.c_int, p, p, p, p]
        L.orc_reorder_range.restype = p
        L.orc_reorder_range.argtypes = [p, i64, i64, ctypes.c_int, ctypes.c_int,
                                        ctypes.c_int, ctypes.c_int]
        L.orc_format_sizes.restype = None
        L.orc_format_sizes.argtypes = [p, p]
        L.orc_format_copy.restype = None
        L.orc_format_copy.argtypes = [p] * 11
        L.orc_format_free.restype = None
        L.orc_format_free.argtypes = [p]
        L.orc_row_cluster.restype = ctypes.c_int
        L.orc_row_cluster.argtypes = [p, i64, i64, p]
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _bits(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x)
    if x.dtype == np.float16:
        x = x.view(np.uint16)
    if x.dtype != np.uint16:
        raise TypeError("expected fp16 values or uint16 fp16 bit patterns")
    return x


def half_to_double(h: int) -> float:
    return lib().orc_half_to_double(int(h) & 0xFFFF)


def spmm(A, B, rows=None):
    """O1: C = A.B over the nonzeros of A, fp64 accumulation, plus
    Mabs = |A|.|B| for the parity tolerance |C - C_ref| <= 1e-2*Mabs + 1e-3.
    ``rows`` (optional) restricts the computation to those rows of A."""
    A, B = _bits(A), _bits(B)
    M, K = A.shape
    K2, N = B.shape
    assert K == K2
    if rows is None:
        r, nr, rp = None, M, None
    else:
        r = np.ascontiguousarray(np.asarray(rows, dtype=np.int64))
        nr, rp = len(r), _ptr(r)
    C = np.empty((nr, N), dtype=np.float64)
    Mabs = np.empty((nr, N), dtype=np.float64)
    rc = lib().orc_spmm(_ptr(A), M, K, _ptr(B), N, rp, nr, _ptr(C), _ptr(Mabs))
    if rc:
        raise ValueError(f"orc_spmm failed ({rc})")
    return C, Mabs


def tile_reorder(masks, cols, W=16, G=4, Z=2):
    """Alg. 1 + reorder retry on one tile.

    masks: W python ints (row bitmasks, row r = bit r, P <= 256 rows)
    cols : W column ids (PAD = -1)
    Returns (perm, cols_after, evicted)."""
    m = np.zeros(4 * W, dtype=np.uint64)
    for j, x in enumerate(masks):
        for w in range(4):
            m[4 * j + w] = np.uint64((int(x) >> (64 * w)) & ((1 << 64) - 1))
    c = np.ascontiguousarray(np.asarray(cols, dtype=np.int32))
    perm = np.zeros(W, dtype=np.uint8)
    ev = np.zeros(16, dtype=np.int32)
    nev = ctypes.c_int(0)
    rc = lib().orc_tile_reorder(_ptr(m), W, G, Z, _ptr(c), _ptr(perm), _ptr(ev),
                                ctypes.byref(nev))
    if rc:
        raise ValueError(f"orc_tile_reorder failed ({rc})")
    return perm.tolist(), c.tolist(), ev[: nev.value].tolist()


@dataclass
class Format:
    """Canonical CR1 arrays.  Tiles of all panels are stored
    consecutively; panel p owns tiles tile_off[p] : tile_off[p] + T[p]."""
    M: int
    K: int
    P: int
    mode: int
    panels: range
    T: np.ndarray          # [npanels] int64
    D: np.ndarray          # [npanels] int64
    col_idx: np.ndarray    # [ntiles, 16] int32, PAD = -1
    perm: np.ndarray       # [ntiles, 16] uint8
    vals: np.ndarray       # [ntiles, P, 8] uint16 (fp16 bits)
    meta: np.ndarray       # [ntiles, P] uint16 (nibble q = i0 + 4*i1 at bits 4q)
    kind: np.ndarray       # [ntiles] uint8 (0 MAIN, 1 OVERFLOW)
    nevict: np.ndarray     # [ntiles] uint8
    rcol: np.ndarray       # [ndtiles, 16] int32 (DENSE mode)
    dvals: np.ndarray      # [ndtiles, P, 16] uint16 (DENSE mode)
    rowmap: np.ndarray = None  # [M] int32: panel row r is row rowmap[r] of A (identity unless row-clustered)
    # CUDA-core tiles (cuda_core_split): per panel the
    # number of 2:4 tiles moved off the tensor cores, and the nonzeros of their
    # columns as panel-local (row, column, fp16 bits) entries, ordered by row
    # then column; panel p owns entries cc_eoff[p] : cc_eoff[p + 1]
    cc_T: np.ndarray = None     # [npanels] int64
    cc_eoff: np.ndarray = None  # [npanels + 1] int64
    cc_row: np.ndarray = None   # [nent] int32 (row within the panel)
    cc_col: np.ndarray = None   # [nent] int32 (column of A)
    cc_val: np.ndarray = None   # [nent] uint16 (fp16 bits, nonzero)

    @property
    def tile_off(self):
        return np.concatenate([[0], np.cumsum(self.T)]).astype(np.int64)

    @property
    def dtile_off(self):
        return np.concatenate([[0], np.cumsum(self.D)]).astype(np.int64)

    @property
    def cc(self):
        """CUDA-core entries (eoff, row, col, val) as check.check_format takes them."""
        return None if self.cc_eoff is None else (self.cc_eoff, self.cc_row, self.cc_col, self.cc_val)

    @property
    def gather(self):
        """gather[t][j] = col_idx[t][perm[t][j]]."""
        return np.take_along_axis(self.col_idx, self.perm.astype(np.int64), axis=1)


def row_cluster(A) -> np.ndarray:
    """Row order of the row-clustered panels: rows by
    decreasing nonzero count, ties by ascending index (orc_row_cluster)."""
    A = _bits(A)
    M, K = A.shape
    perm = np.zeros(M, np.int32)
    rc = lib().orc_row_cluster(_ptr(A), M, K, _ptr(perm))
    if rc:
        raise ValueError(f"orc_row_cluster failed ({rc})")
    return perm


def reorder(A, P=128, mode=0, panels=None, row_order=0, cc_max_nnz=0) -> Format:
    """O2: canonical reorder CR1 of A (M x K fp16), panels of P rows.
    mode 0 = SPTC (paper), 1 = DENSE residual.  ``panels`` = (p0, p1) restricts
    the work to a contiguous panel range (panels are independent).  row_order 1:
    row-clustered panels -- CR1 of A[row_cluster(A)], rowmap = that order.
    cc_max_nnz > 0: then cuda_core_split(format, cc_max_nnz) (f3)."""
    A = _bits(A)
    rowmap = None
    if row_order:
        rowmap = row_cluster(A)
        A = np.ascontiguousarray(A[rowmap])
    M, K = A.shape
    npan = (M + P - 1) // P
    p0, p1 = (0, npan) if panels is None else panels
    h = lib().orc_reorder_range(_ptr(A), M, K, P, mode, p0, p1)
    if not h:
        raise ValueError("orc_reorder_range failed")
    try:
        sz = np.zeros(4, dtype=np.int64)
        lib().orc_format_sizes(h, _ptr(sz))
        npn, nt, nd, P_ = (int(x) for x in sz)
        T = np.zeros(npn, np.int64)
        D = np.zeros(npn, np.int64)
        col_idx = np.zeros((nt, 16), np.int32)
        perm = np.zeros((nt, 16), np.uint8)
        vals = np.zeros((nt, P, 8), np.uint16)
        meta = np.zeros((nt, P), np.uint16)
        kind = np.zeros(nt, np.uint8)
        nevict = np.zeros(nt, np.uint8)
        rcol = np.zeros((nd, 16), np.int32)
        dvals = np.zeros((nd, P, 16), np.uint16)
        lib().orc_format_copy(h, _ptr(T), _ptr(D), _ptr(col_idx), _ptr(perm), _ptr(vals),
                              _ptr(meta), _ptr(kind), _ptr(nevict), _ptr(rcol), _ptr(dvals))
    finally:
        lib().orc_format_free(h)
    f = Format(M, K, P, mode, range(p0, p1), T, D, col_idx, perm, vals, meta, kind,
               nevict, rcol, dvals, rowmap if rowmap is not None else np.arange(M, dtype=np.int32))
    return cuda_core_split(f, A, cc_max_nnz)


def cuda_core_split(f: Format, A, Z: int) -> Format:
    """f3 (§4.7: "For sparser data tile, even with a few
    nonzero elements, using SpTC can result in low resource utilization ...
    we can accelerate the sparser data tiles using CUDA cores").  Reading R-Q28:
    a 2:4 tile of panel p is a CUDA-core tile iff its nonzero count -- the
    nonzeros of A in the panel's rows and the tile's real (non-PAD) columns -- is
    at most Z (Z = 0: none).  CUDA-core tiles leave the tile list (the other
    tiles keep their order and contents); the nonzeros of their columns become
    the panel's CUDA-core entries (panel row, column, fp16 bits), ordered by row,
    then by column.  ``A`` is the matrix the format was built from (A[rowmap]
    for row-clustered panels).  Written as the definition, panel by panel."""
    A = canon_bits(A)
    M = A.shape[0]
    P = f.P
    npan = len(f.T)
    toff = f.tile_off
    keep, ccT, eoff, rows, cols, vals = [], [], [0], [], [], []
    for i, p in enumerate(f.panels):
        r0 = p * P
        nr = min(P, M - r0)
        blk = A[r0:r0 + nr]
        cc_cols = []
        n_cc = 0
        for t in range(toff[i], toff[i + 1]):
            real = [int(c) for c in f.col_idx[t] if c != PAD]
            nnz = int(sum(np.count_nonzero(blk[:, c]) for c in real))
            if Z > 0 and nnz <= Z:
                cc_cols.extend(real)
                n_cc += 1
            else:
                keep.append(t)
        ccT.append(n_cc)
        cc_cols.sort()
        for r in range(nr):
            for c in cc_cols:
                if blk[r, c] != 0:
                    rows.append(r)
                    cols.append(c)
                    vals.append(blk[r, c])
        eoff.append(len(rows))
    keep = np.asarray(keep, dtype=np.int64)
    ccT = np.asarray(ccT, dtype=np.int64)
    f.T = np.asarray(f.T, dtype=np.int64) - ccT
    f.col_idx, f.perm, f.vals, f.meta = f.col_idx[keep], f.perm[keep], f.vals[keep], f.meta[keep]
    f.kind, f.nevict = f.kind[keep], f.nevict[keep]
    f.cc_T = ccT
    f.cc_eoff = np.asarray(eoff, dtype=np.int64)
    f.cc_row = np.asarray(rows, dtype=np.int32)
    f.cc_col = np.asarray(cols, dtype=np.int32)
    f.cc_val = np.asarray(vals, dtype=np.uint16)
    assert len(f.cc_eoff) == npan + 1
    return f


def canon_bits(A) -> np.ndarray:
    """fp16 bits with -0 mapped to +0 (R-Q3): nonzero iff the value is != 0."""
    A = _bits(A).copy()
    A[(A & 0x7FFF) == 0] = 0
    return A


from .check import check_format, decode, format_bytes, canon  # noqa: E402,F401
