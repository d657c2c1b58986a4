"""GPU parity of the CUDA-core tiles (SURVEY §8(f) f3, §4.7,
DESIGN.md R-Q28; jigsaw_options_t.cc_max_nnz = Z).

  * format: BIT-EXACT against oracle.reorder(..., cc_max_nnz=Z) -- the kept 2:4
    tiles (T_p, col_idx, perm, gather, vals, meta, kind, evictions) and the
    CUDA-core entries (per-panel tile counts, entry offsets, rows, columns,
    values) -- and valid under checker O3; Z is taken at the boundaries of the
    oracle's own per-tile nonzero counts (a tile with exactly Z nonzeros moves);
  * SpMM: C within the north-star tolerance of oracle O1 (the product does not
    depend on where a tile runs), integer-valued inputs bit-exact, on every
    launch shape the epilogue has (grouped / single, split-K cluster, CTA pairs,
    k-range pieces, column slices, 32-column tiles, fp32 C, row-clustered
    panels, DENSE residual mode)."""
import numpy as np
import pytest

import oracle
import synth
from oracle import check

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from test_gpu_parity import _dev, _host, assert_format_equal, int_exact, spmm_check  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.set_device(0)


@pytest.fixture
def override():
    yield jig.set_launch_override
    jig.set_launch_override()


def tile_nnz(A, f: oracle.Format):
    """Nonzeros of every tile of an oracle format (panel rows x real columns)."""
    A = oracle.canon_bits(A)
    out = []
    toff = f.tile_off
    for i, p in enumerate(f.panels):
        blk = A[p * f.P:(p + 1) * f.P]
        for t in range(toff[i], toff[i + 1]):
            cols = [int(c) for c in f.col_idx[t] if c != oracle.PAD]
            out.append(int(np.count_nonzero(blk[:, cols])) if cols else 0)
    return np.asarray(out)


def assert_cc_equal(g: dict, ref: oracle.Format):
    assert np.array_equal(g["cc_T"], ref.cc_T)
    assert np.array_equal(g["cc_eoff"], ref.cc_eoff)
    for k in ("cc_row", "cc_col", "cc_val"):
        a, b = g[k], getattr(ref, k)
        assert a.shape == b.shape, k
        assert np.array_equal(a, b), f"{k} differs at {np.argwhere(a != b)[:5].tolist()}"


def build_and_check(A, v, Z, P=128, mode=0, row_order=0, **kw):
    h = jig.reorder(_dev(A), v, panel_rows=P, residual_mode=mode, row_order=row_order, cc_max_nnz=Z, **kw)
    g = h.export()
    ref = oracle.reorder(A, P=P, mode=mode, row_order=row_order, cc_max_nnz=Z)
    assert_format_equal(g, ref)
    assert_cc_equal(g, ref)
    Ap = A if not row_order else A[ref.rowmap]
    D = g["D"] if mode else None
    check.check_format(Ap, P, g["T"], g["gather"], g["vals"], g["meta"], perm=g["perm"], D=D,
                       rcol=g["rcol"] if mode else None, dvals=g["dvals"] if mode else None,
                       cc=(g["cc_eoff"], g["cc_row"], g["cc_col"], g["cc_val"]))
    inf = h.info()
    assert inf["cc_max_nnz"] == Z
    assert inf["cc_tiles"] == int(ref.cc_T.sum())
    assert inf["cc_entries"] == len(ref.cc_row)
    assert inf["ntiles"] == int(ref.T.sum())
    assert inf["evictions"] == int(ref.nevict.sum())
    assert inf["overflow_tiles"] == int((ref.kind == 1).sum())
    return h, ref


CASES = [
    # M, K, v, s, N, kind, seed
    (256, 2048, 8, 0.98, 256, "uniform", 11),  # sparse partial last tiles
    (384, 640, 4, 0.90, 136, "skewed", 12),
    (256, 512, 8, 0.50, 128, "uniform", 13),   # overflow-heavy
    (200, 300, 4, 0.85, 72, "uniform", 14),    # ragged M, K % 16 != 0, N % 32 != 0
]


@pytest.mark.parametrize("M,K,v,s,N,kind,seed", CASES)
def test_cc_thresholds_bit_exact_and_spmm(M, K, v, s, N, kind, seed):
    """Z at the boundaries of the tiles' nonzero counts: the smallest count (and
    one below it: nothing moves), the median, and the largest (every tile moves:
    the product runs on CUDA cores only)."""
    A = synth.vector_sparse(M, K, v, s, seed, kind=kind)
    B = synth.dense_b(K, N, seed)
    cnt = np.sort(tile_nnz(A, oracle.reorder(A, P=128)))
    for Z in sorted({max(int(cnt[0]) - 1, 0), int(cnt[0]), int(cnt[len(cnt) // 2]), int(cnt[-1])}):
        if Z == 0:
            continue
        h, ref = build_and_check(A, v, Z)
        if Z == cnt[-1]:
            assert int(ref.T.sum()) == 0
        C = _host(h.spmm(_dev(B)))
        torch.cuda.synchronize()
        spmm_check(C, A, B)


@pytest.mark.parametrize("ov", [
    {}, dict(tile_n=32, split_k=1), dict(tile_n=64, split_k=2), dict(split_k=4), dict(split_k=8),
    dict(tile_n=128), dict(tile_n=256),
])
def test_cc_single_product_launch_shapes(ov, override):
    """Every single-product launch shape (tile widths, split-K clusters with the
    DSMEM reduce-scatter: the entries are added by the owner CTA of each row)."""
    M, K, v, s, N = 384, 1024, 4, 0.9, 200
    A = synth.vector_sparse(M, K, v, s, 21)
    B = synth.dense_b(K, N, 21)
    cnt = np.sort(tile_nnz(A, oracle.reorder(A, P=128)))
    Z = int(cnt[len(cnt) // 3])
    override(**ov)
    h, _ = build_and_check(A, v, Z)
    spmm_check(_host(h.spmm(_dev(B))), A, B)
    if "split_k" in ov:
        assert jig.last_launch()["split_k"] == ov["split_k"]
    Ai = synth.vector_sparse(M, K, v, s, 22, kind="int")
    Bi = synth.dense_b(K, N, 22, kind="int")
    cnti = np.sort(tile_nnz(Ai, oracle.reorder(Ai, P=128)))
    hi, _ = build_and_check(Ai, v, int(cnti[len(cnti) // 2]))
    Ci = _host(hi.spmm(_dev(Bi)))
    torch.cuda.synchronize()
    int_exact(Ci, Ai, Bi)


@pytest.mark.parametrize("nt", [0, 128, 256])
def test_cc_pair_panels(nt, override):
    """256-row panels on CTA pairs: each CTA adds the entries of its 128 rows."""
    M, K, v, s, N = 520, 768, 8, 0.9, 264
    A = synth.vector_sparse(M, K, v, s, 31)
    B = synth.dense_b(K, N, 31)
    cnt = np.sort(tile_nnz(A, oracle.reorder(A, P=256)))
    if nt:
        override(tile_n=nt)
    h, _ = build_and_check(A, v, int(cnt[len(cnt) // 2]), P=256)
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    assert jig.last_launch()["cta_pair"] == 1
    spmm_check(C, A, B)
    Ai = synth.vector_sparse(M, K, v, s, 32, kind="int")
    Bi = synth.dense_b(K, N, 32, kind="int")
    hi, _ = build_and_check(Ai, v, int(cnt[-1]), P=256, c_dtype=jig.C_F32)
    Ci = _host(hi.spmm(_dev(Bi)))
    torch.cuda.synchronize()
    int_exact(Ci, Ai, Bi)


@pytest.mark.parametrize("pieces", ["nsplit", "kpieces", "off"])
def test_cc_grouped_batch(pieces, override):
    """A grouped launch mixing handles with and without CUDA-core tiles, long
    units cut into column slices or k-range pieces (the last piece adds the
    entries once), against the oracle; integers bit-exact."""
    if pieces == "off":
        override(no_pieces=1)
    elif pieces == "kpieces":
        override(k_pieces=1)
    mats = [synth.vector_sparse(512, 6000, 2, 0.5, 601, kind="int"),
            synth.vector_sparse(300, 3000, 4, 0.9, 603)]
    Bs = [synth.dense_b(6000, 200, 602, kind="int"), synth.dense_b(3000, 136, 604)]
    for i in range(12):
        mats.append(synth.vector_sparse(256, 512, 8, 0.95, 610 + i))
        Bs.append(synth.dense_b(512, 64, 630 + i))
    hs = []
    for i, a in enumerate(mats):
        cnt = np.sort(tile_nnz(a, oracle.reorder(a, P=128)))
        Z = 0 if i % 3 == 2 else int(cnt[len(cnt) // 4])
        hs.append(jig.reorder(_dev(a), 2 if i == 0 else (4 if i == 1 else 8), cc_max_nnz=Z))
    dB = [_dev(b) for b in Bs]
    for rep in range(2):
        dC = [torch.full((a.shape[0], b.shape[1]), 7.0, dtype=torch.float16, device="cuda")
              for a, b in zip(mats, Bs)]
        jig.spmm_batched(hs, dB, dC)
        torch.cuda.synchronize()
        d = jig.last_launch()
        assert (d["split_slots"] > 0) == (pieces == "kpieces"), d
        for i, (a, b, c) in enumerate(zip(mats, Bs, dC)):
            if i == 0:
                int_exact(_host(c), a, b)
            else:
                spmm_check(_host(c), a, b)


@pytest.mark.parametrize("P,mode", [(128, 0), (256, 0), (128, 1)])
def test_cc_row_clustered_and_dense_mode(P, mode, override):
    """Row-clustered panels (the entries belong to rows of A[rowmap], C rows are
    scattered back) and the DENSE residual mode (dense tiles are not affected)."""
    M, K, v, s = 512, 640, 4, 0.8
    A = synth.vector_sparse(M, K, v, s, 41, kind="skewed")
    B = synth.dense_b(K, 136, 41)
    ref0 = oracle.reorder(A, P=P, mode=mode, row_order=1)
    cnt = np.sort(tile_nnz(A[ref0.rowmap], ref0))
    Z = int(cnt[len(cnt) // 2])
    h, ref = build_and_check(A, v, Z, P=P, mode=mode, row_order=1)
    assert int(ref.cc_T.sum()) > 0
    spmm_check(_host(h.spmm(_dev(B))), A, B)
    hz, _ = build_and_check(A, v, Z, P=P, mode=mode)
    spmm_check(_host(hz.spmm(_dev(B))), A, B)


def test_cc_all_tiles_and_empty_panels():
    """Z = everything: every panel runs on CUDA cores only (T_p = 0, the
    accumulator is never touched by the tensor cores); all-zero panels have no
    entries and are written as zeros over a pre-filled C."""
    M, K, N = 640, 300, 96
    A = synth.vector_sparse(M, K, 4, 0.95, 51)
    A[128:256] = 0
    B = synth.dense_b(K, N, 51)
    h, ref = build_and_check(A, 4, 1 << 20)
    assert int(ref.T.sum()) == 0 and ref.cc_T.sum() > 0
    C = torch.full((M, N), 5.0, dtype=torch.float16, device="cuda")
    h.spmm(_dev(B), C)
    torch.cuda.synchronize()
    Ch = _host(C)
    assert np.all(Ch[128:256] == 0)
    spmm_check(Ch, A, B)
