"""Pins for oracle O1 (naive SpMM) and its fp16 decoding.

Each test checks the oracle against something other than itself: the numpy
float16 decoder (exhaustive), exact integer arithmetic, a closed form (A = I),
a library matmul for the dense special case, and exact rational brute force."""
from fractions import Fraction

import numpy as np
import pytest

import oracle
import synth


def test_half_decode_exhaustive():
    """All 65536 fp16 bit patterns decode exactly as numpy's IEEE binary16."""
    bits = np.arange(65536, dtype=np.uint32).astype(np.uint16)
    ref = bits.view(np.float16).astype(np.float64)
    got = np.array([oracle.half_to_double(int(b)) for b in bits])
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(got), nan)
    assert np.array_equal(got[~nan], ref[~nan])
    # sign of zero is preserved too
    assert np.signbit(got[0x8000]) and not np.signbit(got[0])


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_integer_valued_exact(seed):
    """A in {+-1,+-2}, B in {-2..2}: every partial sum is an integer, so the
    result is exact and equals the int64 product."""
    A = synth.vector_sparse(64, 96, 4, 0.7, seed, kind="int")
    B = synth.dense_b(96, 40, seed, kind="int")
    C, _ = oracle.spmm(A, B)
    ref = A.view(np.float16).astype(np.int64) @ B.view(np.float16).astype(np.int64)
    assert np.array_equal(C, ref.astype(np.float64))


def test_identity_gives_B():
    """Closed form: A = I  =>  C = B exactly, Mabs = |B|."""
    K = 48
    A = np.eye(K, dtype=np.float16).view(np.uint16)
    B = synth.dense_b(K, 24, 5)
    C, Mabs = oracle.spmm(A, B)
    Bf = B.view(np.float16).astype(np.float64)
    assert np.array_equal(C, Bf)
    assert np.array_equal(Mabs, np.abs(Bf))


def test_dense_equals_library_matmul():
    """s = 0: every entry of A is a nonzero, the sum is over all k; fp64 matmul
    of the same fp16 inputs agrees to fp64 rounding."""
    A = synth.vector_sparse(32, 64, 1, 0.0, 9)
    B = synth.dense_b(64, 16, 9)
    C, Mabs = oracle.spmm(A, B)
    Af, Bf = A.view(np.float16).astype(np.float64), B.view(np.float16).astype(np.float64)
    assert np.allclose(C, Af @ Bf, rtol=0, atol=1e-12)
    assert np.allclose(Mabs, np.abs(Af) @ np.abs(Bf), rtol=0, atol=1e-12)


def test_brute_force_tiny_exact_rationals():
    """M, K, N <= 6: exact rational sum of products (fp16 values are dyadic)."""
    rng = np.random.default_rng(11)
    for _ in range(20):
        M, K, N = rng.integers(1, 7, size=3)
        A = (rng.uniform(-2, 2, size=(M, K)) * (rng.random((M, K)) < 0.5)).astype(np.float16)
        B = rng.uniform(-2, 2, size=(K, N)).astype(np.float16)
        C, _ = oracle.spmm(A, B)
        for i in range(M):
            for n in range(N):
                s = sum((Fraction(float(A[i, k])) * Fraction(float(B[k, n])) for k in range(K)),
                        Fraction(0))
                assert abs(Fraction(C[i, n]) - s) <= abs(s) * Fraction(1, 2 ** 50)


def test_zero_entries_are_skipped():
    """The sparse definition multiplies only the nonzeros of A (R-Q3): a -0 or +0
    entry of A times an Inf/NaN of B contributes nothing."""
    A = np.array([[0.0, -0.0, 1.0]], dtype=np.float16)
    B = np.array([[np.inf], [np.nan], [2.0]], dtype=np.float16)
    C, _ = oracle.spmm(A, B)
    assert C[0, 0] == 2.0


def test_row_subset_matches_full():
    A = synth.vector_sparse(128, 64, 8, 0.8, 3)
    B = synth.dense_b(64, 32, 3)
    C, M1 = oracle.spmm(A, B)
    rows = [5, 127, 0, 64]
    Cs, Ms = oracle.spmm(A, B, rows=rows)
    assert np.array_equal(Cs, C[rows]) and np.array_equal(Ms, M1[rows])
