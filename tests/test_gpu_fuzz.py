"""Seeded randomised GPU parity sweep over the option / launch-shape matrix:
shape (ragged M, K, N), v, sparsity, mask kind, panel height, residual mode,
C element type, row order, and a forced launch shape (tile width, split-K,
piece mode), and (for half the seeds) a CUDA-core threshold cc_max_nnz taken
from the configuration's own tile nonzero counts -- each configuration's format
bit-exact against the oracle on a
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
from test_gpu_cuda_core import tile_nnz  # noqa: E402


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
    ref = oracle.reorder(A, P=P, mode=mode, row_order=row_order)
    Ap = A[ref.rowmap] if row_order else A
    Z = 0  # CUDA-core threshold (f3), from a separate stream so the other draws stay as they were
    rc = np.random.default_rng(5000 + seed)
    if rc.random() < 0.5 and int(ref.T.sum()) > 0:
        cnt = np.sort(tile_nnz(Ap, ref))
        Z = max(1, int(cnt[int(rc.integers(0, len(cnt)))]))
    h = jig.reorder(_dev(A), v, panel_rows=P, residual_mode=mode, c_dtype=c_dtype, row_order=row_order,
                    cc_max_nnz=Z)
    g = h.export()
    npan = (M + P - 1) // P
    p = seed % npan
    assert np.array_equal(g["rowmap"], ref.rowmap)
    sub = oracle.reorder(Ap, P=P, mode=mode, panels=(p, p + 1), cc_max_nnz=Z)
    assert_format_equal(g, sub, panels=(p, p + 1))
    assert g["cc_T"][p] == sub.cc_T[0]
    e0, e1 = int(g["cc_eoff"][p]), int(g["cc_eoff"][p + 1])
    for k in ("cc_row", "cc_col", "cc_val"):
        assert np.array_equal(g[k][e0:e1], getattr(sub, k)), k
    with jig.launch_override(**ov):
        C = h.spmm(_dev(B))
        torch.cuda.synchronize()
    Ch = _host(C)
    if kind == "int" and c_dtype == 1:
        int_exact(Ch, A, B)
    else:
        spmm_check(Ch, A, B)
