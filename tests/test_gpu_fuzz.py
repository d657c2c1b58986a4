"""Seeded randomised GPU parity sweep over the option / launch-shape matrix:
shape (ragged M, K, N), v, sparsity, mask kind, panel height, residual mode,
C element type, row order, and a forced launch shape (tile width, split-K,
piece mode) -- each configuration's format bit-exact against the oracle on a
sampled panel and C within the north-star tolerance (integer inputs: exact).
The interactions of the options, not each option alone (tested elsewhere)."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from test_gpu_parity import _dev, _host, assert_format_equal, int_exact, spmm_check  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.set_device(0)


def _config(seed):
    rng = np.random.default_rng(1000 + seed)
    v = int(rng.choice([1, 2, 4, 8]))
    P = int(rng.choice([128, 128, 256]))
    M = int(rng.integers(1, 7)) * 96 + int(rng.integers(0, 4)) * v + v
    M -= M % v
    K = int(rng.integers(40, 900))
    N = 8 * int(rng.integers(1, 40))
    s = float(rng.choice([0.5, 0.7, 0.85, 0.95, 0.99]))
    kind = str(rng.choice(["uniform", "skewed", "int"]))
    mode = int(rng.integers(0, 2))
    c_dtype = int(rng.integers(0, 2))
    row_order = int(rng.integers(0, 2))
    ov = [{}, {"tile_n": 32, "split_k": 2}, {"tile_n": 64, "split_k": 4}, {"tile_n": 128}, {"tile_n": 256},
          {"k_pieces": 1}, {"no_pieces": 1}][int(rng.integers(0, 7))]
    if P == 256:
        ov = {k: x for k, x in ov.items() if k != "split_k"}
    return M, K, N, v, s, kind, P, mode, c_dtype, row_order, ov


@pytest.mark.parametrize("seed", range(40))
def test_fuzz_options(seed):
    M, K, N, v, s, kind, P, mode, c_dtype, row_order, ov = _config(seed)
    A = synth.vector_sparse(M, K, v, s, 3000 + seed, kind=kind)
    B = synth.dense_b(K, N, 3000 + seed, kind="int" if kind == "int" else "uniform")
    h = jig.reorder(_dev(A), v, panel_rows=P, residual_mode=mode, c_dtype=c_dtype, row_order=row_order)
    g = h.export()
    npan = (M + P - 1) // P
    p = seed % npan
    ref = oracle.reorder(A, P=P, mode=mode, row_order=row_order)
    assert np.array_equal(g["rowmap"], ref.rowmap)
    assert_format_equal(g, oracle.reorder(A[ref.rowmap] if row_order else A, P=P, mode=mode, panels=(p, p + 1)),
                        panels=(p, p + 1))
    with jig.launch_override(**ov):
        C = h.spmm(_dev(B))
        torch.cuda.synchronize()
    Ch = _host(C)
    if kind == "int" and c_dtype == 1:
        int_exact(Ch, A, B)
    else:
        spmm_check(Ch, A, B)
