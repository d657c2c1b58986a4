"""Pins of the row-clustered panel order (DESIGN.md R-Q27):
oracle.row_cluster(A) must be THE order "rows by decreasing nonzero count, ties
by ascending index" -- pinned by the invariants that characterise that order
uniquely, by brute force over all permutations of tiny matrices, and by the
structure of vector-sparse rows; and CR1 applied to A[order] must be a valid
format of A[order] (checker O3)."""
import itertools

import numpy as np
import pytest

import oracle
import synth
from oracle import check


def _nnz(A):
    return ((A & 0x7FFF) != 0).sum(axis=1)


@pytest.mark.parametrize("M,K,v,s,kind,seed", [
    (256, 192, 1, 0.9, "uniform", 1), (512, 256, 4, 0.8, "skewed", 2), (384, 100, 8, 0.95, "skewed", 3),
    (200, 64, 2, 0.99, "uniform", 4)])
def test_row_cluster_invariants(M, K, v, s, kind, seed):
    A = synth.vector_sparse(M, K, v, s, seed, kind=kind)
    A[7] = 0x8000                                   # a row of -0 only: zero count (R-Q3)
    p = oracle.row_cluster(A)
    assert sorted(p.tolist()) == list(range(M))     # a permutation
    c = _nnz(A)[p]
    assert np.all(np.diff(c) <= 0)                  # non-increasing counts
    same = np.diff(c) == 0
    assert np.all(np.diff(p)[same] > 0)             # equal counts: ascending row index
    assert p[-1] == max(r for r in range(M) if _nnz(A)[r] == 0)


def test_row_cluster_brute_force_tiny():
    rng = np.random.default_rng(0)
    for trial in range(40):
        M, K = int(rng.integers(1, 6)), int(rng.integers(1, 6))
        A = np.where(rng.random((M, K)) < 0.5, np.uint16(0x3C00), np.uint16(0)).astype(np.uint16)
        cnt = _nnz(A)
        good = [q for q in itertools.permutations(range(M))
                if all(cnt[q[i]] > cnt[q[i + 1]] or (cnt[q[i]] == cnt[q[i + 1]] and q[i] < q[i + 1])
                       for i in range(M - 1))]
        assert len(good) == 1
        assert oracle.row_cluster(A).tolist() == list(good[0])


@pytest.mark.parametrize("v", [2, 4, 8])
def test_vector_rows_stay_together(v):
    """The v rows of a nonzero vector (R-Q1) share their support, so they
    keep adjacent, in order, in the clustered order."""
    A = synth.vector_sparse(512, 300, v, 0.85, 10 + v, kind="skewed")
    p = oracle.row_cluster(A)
    for i in range(0, 512, v):
        assert p[i] % v == 0 and np.array_equal(p[i:i + v], p[i] + np.arange(v))


@pytest.mark.parametrize("P,mode", [(128, 0), (256, 0), (128, 1)])
def test_clustered_format_is_a_valid_format_of_permuted_a(P, mode):
    A = synth.vector_sparse(512, 256, 4, 0.8, 21, kind="skewed")
    f = oracle.reorder(A, P=P, mode=mode, row_order=1)
    assert np.array_equal(f.rowmap, oracle.row_cluster(A))
    Ap = A[f.rowmap]
    check.check_format(Ap, P, f.T, f.gather, f.vals, f.meta, perm=f.perm,
                       D=f.D if mode else None, rcol=f.rcol if mode else None, dvals=f.dvals if mode else None)
    g = oracle.reorder(Ap, P=P, mode=mode)          # CR1 of the permuted matrix, by definition
    for k in ("T", "col_idx", "perm", "vals", "meta"):
        assert np.array_equal(getattr(f, k), getattr(g, k)), k
