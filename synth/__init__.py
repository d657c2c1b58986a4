"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and
bench.py.  This module holds NONE of the method's arithmetic (no reorder, no
compression, no product): it only draws vector-sparse fp16 matrices and dense
fp16 right-hand sides with the structure of the paper's workloads.

Recipe ("replacing each nonzero element with a
1-D vector", P:289 DLMC random pruning at exact sparsity; R-Q1, R-Q2):
  * A is M x K; the vector grid is (M/v) x K; a nonzero cell of the grid is a
    v x 1 column vector (rows v*i .. v*i+v-1 of column k);
  * exactly round((1-s) * (M/v) * K) cells are nonzero, chosen without
    replacement ("uniform"), or with per-vector-row weights drawn from a Beta
    distribution ("skewed", mimics magnitude-pruned DLMC rows);
  * each element of a nonzero vector is fp16_RN(u), u ~ U(-1, 1) with |u|
    clamped to >= 2^-6, so no vector element is zero;
  * "int": A in {+-1, +-2}, B in {-2..2} (exact in fp16/fp32 for any order);
  * B is fp16_RN(U(-1, 1)).
All generators take an integer seed and use numpy's PCG64 (default_rng).
"""
from __future__ import annotations

import numpy as np

SEED_BASE = 0x4A16 * 1000


def vector_mask(M: int, K: int, v: int, s: float, seed: int, kind: str = "uniform") -> np.ndarray:
    """Boolean (M/v) x K grid of nonzero vectors at exact sparsity s."""
    if M % v:
        raise ValueError("M must be a multiple of v")
    rng = np.random.default_rng(seed)
    mv = M // v
    ncell = mv * K
    nnz = int(round((1.0 - s) * ncell))
    grid = np.zeros(ncell, dtype=bool)
    if kind in ("uniform", "int"):
        grid[rng.choice(ncell, size=nnz, replace=False)] = True
    elif kind == "skewed":
        w = rng.beta(0.7, 2.0, size=mv) + 1e-3
        keys = np.log(np.repeat(w, K)) + rng.gumbel(size=ncell)   # weighted sampling w/o replacement
        if nnz:
            grid[np.argpartition(-keys, nnz - 1)[:nnz]] = True
    else:
        raise ValueError(kind)
    return grid.reshape(mv, K)


def vector_sparse(M: int, K: int, v: int, s: float, seed: int, kind: str = "uniform") -> np.ndarray:
    """M x K fp16 (returned as uint16 bit patterns) vector-sparse matrix."""
    grid = vector_mask(M, K, v, s, seed, kind)
    rng = np.random.default_rng(seed + 7919)
    full = np.repeat(grid, v, axis=0)
    if kind == "int":
        vals = rng.choice(np.array([-2.0, -1.0, 1.0, 2.0]), size=(M, K))
    else:
        u = rng.uniform(-1.0, 1.0, size=(M, K))
        u = np.where(np.abs(u) < 2.0 ** -6, np.copysign(2.0 ** -6, u), u)
        vals = u
    A = np.where(full, vals, 0.0).astype(np.float16)
    return A.view(np.uint16)


def dense_b(K: int, N: int, seed: int, kind: str = "uniform") -> np.ndarray:
    """K x N dense fp16 right-hand side (uint16 bit patterns)."""
    rng = np.random.default_rng(seed + 104729)
    if kind == "int":
        B = rng.integers(-2, 3, size=(K, N)).astype(np.float16)
    else:
        B = rng.uniform(-1.0, 1.0, size=(K, N)).astype(np.float16)
    return B.view(np.uint16)


def nm24(M: int, K: int, seed: int) -> np.ndarray:
    """Already-2:4 matrix: every row keeps exactly 2 of each aligned 4 columns
    (the P:337 "pruned matrices ... computed directly without reordering" case)."""
    if K % 4:
        raise ValueError("K must be a multiple of 4")
    rng = np.random.default_rng(seed)
    keep = np.zeros((M, K // 4, 4), dtype=bool)
    pick = np.argsort(rng.random((M, K // 4, 4)), axis=2)[:, :, :2]
    np.put_along_axis(keep, pick, True, axis=2)
    u = rng.uniform(0.25, 1.0, size=(M, K)) * rng.choice([-1.0, 1.0], size=(M, K))
    return np.where(keep.reshape(M, K), u, 0.0).astype(np.float16).view(np.uint16)


def venom(M: int, K: int, V: int, Mb: int, seed: int, kind: str = "uniform") -> np.ndarray:
    """VENOM-style V:2:Mb matrix (the "pruned matrices ... computed directly
    without reordering" of P:321-337 §4.5, Table 3): rows in
    blocks of V, columns in blocks of Mb; in every V x Mb block 4 columns are
    selected (the same for all V rows of the block) and every row keeps 2 of
    those 4 (2:4), so the density is 2 / Mb.  A last, narrower column block
    selects min(4, width) columns and keeps min(2, that) per row.  Values as in
    vector_sparse.  With 4 | Mb every aligned group of 4 columns lies inside one
    block, so the matrix is natively 2:4 (what cuSPARSELt accepts)."""
    if M % V:
        raise ValueError("M must be a multiple of V")
    rng = np.random.default_rng(seed)
    keep = np.zeros((M, K), dtype=bool)
    for r0 in range(0, M, V):
        for c0 in range(0, K, Mb):
            w = min(Mb, K - c0)
            sel = c0 + np.sort(rng.choice(w, size=min(4, w), replace=False))
            nk = min(2, len(sel))
            pick = np.argsort(rng.random((V, len(sel))), axis=1)[:, :nk]
            keep[r0 + np.arange(V)[:, None], sel[pick]] = True
    rv = np.random.default_rng(seed + 7919)
    if kind == "int":
        vals = rv.choice(np.array([-2.0, -1.0, 1.0, 2.0]), size=(M, K))
    else:
        u = rv.uniform(-1.0, 1.0, size=(M, K))
        vals = np.where(np.abs(u) < 2.0 ** -6, np.copysign(2.0 ** -6, u), u)
    return np.where(keep, vals, 0.0).astype(np.float16).view(np.uint16)


# --- the paper's workload families (BASELINE.json configs) ---------

C1 = dict(M=256, K=256, v=4, s=0.80, N=64)

C2_SHAPES = [(512, 2048), (2048, 512)]
C2_V = [2, 4, 8]
C2_S = [0.50, 0.70, 0.80, 0.90, 0.95, 0.98]
C2_N = 256

C3_SHAPES = [(64, 64), (64, 576), (256, 64), (64, 256), (128, 256), (128, 1152), (512, 128),
             (512, 256), (128, 512), (256, 512), (256, 2304), (1024, 256), (1024, 512),
             (256, 1024), (512, 1024), (512, 4608), (2048, 512), (2048, 1024), (512, 2048)]
C3_V = [4, 8]
C3_S = [0.70, 0.80, 0.90, 0.95]
C3_N = [256, 1024]

C4_SHAPES = [(4096, 4096), (11008, 4096)]
C4_S = [0.50, 0.70, 0.80, 0.90]
C4_N = 2048


def c2_points():
    """The 36 (M, K, v, s, N) points of configs[1] (DLMC transformer, N=256)."""
    return [(M, K, v, s, C2_N) for (M, K) in C2_SHAPES for v in C2_V for s in C2_S]


# f4 (Table 3): V:2:Mb matrices, V in {32, 64, 128}, block
# widths Mb = 12 / 20 / 40 / 100 (sparsity 83.3 / 90 / 95 / 98 %; 4 | Mb so each
# matrix is natively 2:4 for the cuSPARSELt baseline), Llama-shaped 4096 x 4096,
# N = 2048
VENOM_SHAPE = (4096, 4096)
VENOM_V = [32, 64, 128]
VENOM_MB = [12, 20, 40, 100]
VENOM_N = 2048


def venom_points():
    """(M, K, V, Mb, N) of the f4 workload."""
    M, K = VENOM_SHAPE
    return [(M, K, V, mb, VENOM_N) for V in VENOM_V for mb in VENOM_MB]


def c4_points():
    return [(M, K, 8, s, C4_N) for (M, K) in C4_SHAPES for s in C4_S]
