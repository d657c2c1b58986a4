"""The seeded generators produce the structure DESIGN.md §4 states."""
import numpy as np
import pytest

import synth


@pytest.mark.parametrize("v", [1, 2, 4, 8])
@pytest.mark.parametrize("kind", ["uniform", "skewed", "int"])
def test_vector_structure_and_exact_sparsity(v, kind):
    M, K, s = 128, 96, 0.8
    A = synth.vector_sparse(M, K, v, s, 3, kind=kind)
    nz = (A & 0x7FFF) != 0
    grid = nz.reshape(M // v, v, K)
    # a vector is all-nonzero or all-zero (no zero element inside a vector)
    assert np.all(grid.all(axis=1) == grid.any(axis=1))
    assert grid.any(axis=1).sum() == round((1 - s) * (M // v) * K)
    if kind == "int":
        assert set(np.unique(A.view(np.float16)[nz]).tolist()) <= {-2.0, -1.0, 1.0, 2.0}
    else:
        vals = np.abs(A.view(np.float16)[nz].astype(np.float64))
        assert vals.min() >= 2.0 ** -6 * (1 - 2 ** -10) and vals.max() <= 1.0


def test_deterministic():
    a = synth.vector_sparse(64, 64, 4, 0.9, 42)
    b = synth.vector_sparse(64, 64, 4, 0.9, 42)
    c = synth.vector_sparse(64, 64, 4, 0.9, 43)
    assert np.array_equal(a, b) and not np.array_equal(a, c)
    assert np.array_equal(synth.dense_b(32, 16, 1), synth.dense_b(32, 16, 1))


def test_nm24_is_24():
    A = synth.nm24(64, 64, 1)
    nz = ((A & 0x7FFF) != 0).reshape(64, 16, 4)
    assert np.all(nz.sum(axis=2) == 2)


def test_workload_lists():
    assert len(synth.c2_points()) == 36
    assert all(M % v == 0 for (M, K, v, s, N) in synth.c2_points())
