"""Pins of the CUDA-core tile split (SURVEY §8(f) f3, §4.7,
DESIGN.md R-Q28): oracle.cuda_core_split moves every 2:4 tile whose nonzero
count is <= Z off the tile list and lists the nonzeros of its columns as
(panel row, column, value) entries ordered by row, then column.

Pinned by a hand-derived example (the boundary Z = nnz of a tile), by the
closed form at Z = max (every tile moves: the entries are the panel's nonzeros
in row-major order, compared with numpy.nonzero), by the boundary of the
threshold on random matrices (a tile with exactly Z nonzeros moves, with Z - 1
it stays), and by the independent checker O3 (bijection onto S_p, entry order,
decode == canon(A)) with fault injection."""
import numpy as np
import pytest

import oracle
import synth
from oracle import check

H1, H2, H3 = 0x3C00, 0x4000, 0xBC00  # fp16 1.0, 2.0, -1.0


def _hand_matrix():
    """16 x 18, P = 16.  Columns 0..15: one nonzero each, at row c (so every
    4-column group has at most one nonzero per row: the first tile takes columns
    0..15 unchanged, 16 nonzeros).  Columns 16 and 17: one nonzero each at rows
    0 and 5 -> the partial last tile {16, 17} + 14 PAD with 2 nonzeros (P:190:
    the remainder of S_p forms the last tile)."""
    A = np.zeros((16, 18), np.uint16)
    for c in range(16):
        A[c, c] = H1
    A[0, 16] = H2
    A[5, 17] = H3
    return A


def test_hand_example_threshold_boundary():
    A = _hand_matrix()
    f0 = oracle.reorder(A, P=16)
    assert list(f0.T) == [2] and f0.cc_T.tolist() == [0] and len(f0.cc_row) == 0
    # Z = 1: no tile has <= 1 nonzero
    f1 = oracle.reorder(A, P=16, cc_max_nnz=1)
    assert list(f1.T) == [2] and len(f1.cc_row) == 0
    # Z = 2: the last tile (2 nonzeros) moves; entries (0, 16, 2.0), (5, 17, -1.0)
    f2 = oracle.reorder(A, P=16, cc_max_nnz=2)
    assert list(f2.T) == [1] and f2.cc_T.tolist() == [1]
    assert f2.cc_row.tolist() == [0, 5] and f2.cc_col.tolist() == [16, 17]
    assert f2.cc_val.tolist() == [H2, H3] and f2.cc_eoff.tolist() == [0, 2]
    assert f2.col_idx.tolist() == f0.col_idx[:1].tolist()
    # Z = 16: both tiles move; entries in row order, then column order
    f16 = oracle.reorder(A, P=16, cc_max_nnz=16)
    assert list(f16.T) == [0] and f16.cc_T.tolist() == [2]
    exp = sorted([(c, c, H1) for c in range(16)] + [(0, 16, H2), (5, 17, H3)])
    got = list(zip(f16.cc_row.tolist(), f16.cc_col.tolist(), f16.cc_val.tolist()))
    assert got == exp
    for f in (f1, f2, f16):
        check.check_format(A, 16, f.T, f.gather, f.vals, f.meta, perm=f.perm, cc=f.cc)


@pytest.mark.parametrize("P", [128, 256])
@pytest.mark.parametrize("M,K,v,s,seed", [(256, 320, 4, 0.9, 1), (384, 200, 2, 0.7, 2), (512, 256, 8, 0.97, 3)])
def test_all_tiles_to_cuda_cores_is_row_major_nonzeros(P, M, K, v, s, seed):
    """Z >= P * 16 (no tile can have more nonzeros): no 2:4 tile is left and the
    entries of panel p are exactly numpy.nonzero of its rows, in row-major order."""
    A = synth.vector_sparse(M, K, v, s, seed)
    A[3, 5] = 0x8000  # -0 is a zero (R-Q3)
    f = oracle.reorder(A, P=P, cc_max_nnz=P * 16)
    assert f.T.sum() == 0 and len(f.col_idx) == 0
    Ac = check.canon(A)
    for p in range((M + P - 1) // P):
        blk = Ac[p * P:(p + 1) * P]
        r, c = np.nonzero(blk)
        e = slice(f.cc_eoff[p], f.cc_eoff[p + 1])
        assert np.array_equal(f.cc_row[e], r) and np.array_equal(f.cc_col[e], c)
        assert np.array_equal(f.cc_val[e], blk[r, c])
    check.check_format(A, P, f.T, f.gather, f.vals, f.meta, perm=f.perm, cc=f.cc)


def _tile_nnz(A, P, f0):
    """nnz of every tile of f0 (numpy, from the tile's real columns)."""
    Ac = check.canon(A)
    out = []
    for p in range(len(f0.T)):
        for t in range(f0.tile_off[p], f0.tile_off[p + 1]):
            cols = [c for c in f0.col_idx[t] if c != -1]
            out.append(int(np.count_nonzero(Ac[p * P:(p + 1) * P][:, cols])))
    return np.array(out)


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("M,K,v,s,seed,P", [(384, 256, 4, 0.95, 11, 128), (512, 200, 2, 0.6, 12, 128),
                                            (512, 300, 8, 0.9, 13, 256)])
def test_threshold_boundary_random(mode, M, K, v, s, seed, P):
    """A tile with exactly Z nonzeros moves at Z and stays at Z - 1; the kept
    tiles are the CR1 tiles with more than Z nonzeros, in their CR1 order."""
    A = synth.vector_sparse(M, K, v, s, seed)
    f0 = oracle.reorder(A, P=P, mode=mode)
    nnz = _tile_nnz(A, P, f0)
    for Z in sorted(set([int(np.median(nnz)), int(nnz.min()), int(nnz.max())])):
        for z in (Z, Z - 1):
            f = oracle.reorder(A, P=P, mode=mode, cc_max_nnz=z)
            kept = np.nonzero(nnz > z)[0] if z > 0 else np.arange(len(nnz))
            assert np.array_equal(f.col_idx, f0.col_idx[kept])
            assert np.array_equal(f.vals, f0.vals[kept]) and np.array_equal(f.meta, f0.meta[kept])
            assert np.array_equal(f.kind, f0.kind[kept]) and np.array_equal(f.nevict, f0.nevict[kept])
            assert f.T.sum() + f.cc_T.sum() == f0.T.sum()
            assert np.array_equal(f.D, f0.D) and np.array_equal(f.rcol, f0.rcol)
            check.check_format(A, P, f.T, f.gather, f.vals, f.meta, perm=f.perm, D=f.D, rcol=f.rcol,
                               dvals=f.dvals, cc=f.cc)


def test_row_clustered_with_cuda_core_tiles():
    A = synth.vector_sparse(512, 256, 4, 0.9, 21, kind="skewed")
    f0 = oracle.reorder(A, P=128, row_order=1)
    Z = int(np.median(_tile_nnz(A[f0.rowmap], 128, f0)))
    f = oracle.reorder(A, P=128, row_order=1, cc_max_nnz=Z)
    assert 0 < f.cc_T.sum() < f0.T.sum()
    Ap = A[f.rowmap]
    check.check_format(Ap, 128, f.T, f.gather, f.vals, f.meta, perm=f.perm, cc=f.cc)


def test_checker_rejects_faulty_entries():
    A = synth.vector_sparse(256, 192, 4, 0.9, 31)
    Z = int(np.median(_tile_nnz(A, 128, oracle.reorder(A, P=128))))
    f = oracle.reorder(A, P=128, cc_max_nnz=Z)
    n = len(f.cc_row)
    assert n > 4
    args = (A, 128, f.T, f.gather, f.vals, f.meta)
    check.check_format(*args, perm=f.perm, cc=f.cc)
    eoff, row, col, val = f.cc
    bad = [
        (np.concatenate([[0], eoff[1:] - 1]).clip(0), row[1:], col[1:], val[1:]),   # an entry dropped
        (eoff, row, col, np.where(np.arange(n) == 2, np.uint16(0x3C01), val)),      # a wrong value
        (eoff, row[::-1].copy(), col[::-1].copy(), val[::-1].copy()),               # order reversed
        (eoff, row, col, np.where(np.arange(n) == 0, np.uint16(0), val)),           # a zero entry
    ]
    for cc in bad:
        with pytest.raises(AssertionError):
            check.check_format(*args, perm=f.perm, cc=cc)
    # a CUDA-core column that is also a tile column
    if len(f.gather):
        g = f.gather.copy()
        t = 0
        j = int(np.nonzero(g[t] != -1)[0][0])
        g[t, j] = col[0]
        with pytest.raises(AssertionError):
            check.check_format(A, 128, f.T, g, f.vals, f.meta, cc=f.cc)
