"""Pins for oracle O2 at matrix level (multi-granularity reorder P:132-190 and
reorder-aware format P:192-206) and for the independent checker O3.

Pinned against: the metadata worked example, closed forms (dense panel,
all-zero panel, already-2:4 input P:337), bounds that follow from the retry
rule, and the independent decoder (decode == canon(A), bijection)."""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from oracle import check


def _check(A, f):
    check.check_format(A, f.P, f.T, f.gather, f.vals, f.meta, perm=f.perm,
                       D=f.D if f.mode == 1 else None,
                       rcol=f.rcol if f.mode == 1 else None,
                       dvals=f.dvals if f.mode == 1 else None,
                       panels=f.panels)


def test_fig3_metadata_example(golden_dir):
    """first row with nonzeros at (0,3) and (1,2) -> metadata nibbles 0xC, 0x9."""
    g = json.load(open(os.path.join(golden_dir, "fig3_metadata.json")))
    A = np.zeros((2, 8), np.float16)
    (a0, a1), (b0, b1) = g["row0_nonzero_positions"]
    A[0, [a0, a1, 4 + b0, 4 + b1]] = 1.0
    A[1, [c for c in range(8) if c not in (a0, a1, 4 + b0, 4 + b1)]] = 1.0  # no all-zero column
    f = oracle.reorder(A, P=2)
    assert f.perm[0].tolist() == list(range(16))          # already 2:4: identity
    meta0 = int(f.meta[0, 0])
    assert [hex(meta0 & 0xF).upper().replace("X", "x"), hex((meta0 >> 4) & 0xF).upper().replace("X", "x")] \
        == g["expected_nibbles"]
    assert meta0 & 0xFF == int(g["expected_row0_meta_low_byte"], 16)
    _check(A, f)


@pytest.mark.parametrize("K", [16, 64, 128])
def test_dense_panel_closed_form(K):
    """s = 0 (SURVEY §8c a3 closed form): every 16-column tile evicts slots 0..7
    and keeps 8..15 with perm [0,1,8,9, 2,3,10,11, 4,5,12,13, 6,7,14,15] and
    nibble (2,3) = 0xE; the last tile has 8 real columns in slots 0..7, nibble
    (0,1) = 0x4; T_p = K/8."""
    P = 16
    A = np.ones((P, K), np.float16)
    f = oracle.reorder(A, P=P)
    assert f.T.tolist() == [K // 8]
    perm = [0, 1, 8, 9, 2, 3, 10, 11, 4, 5, 12, 13, 6, 7, 14, 15]
    for t in range(K // 8):
        assert f.perm[t].tolist() == perm
        last = t == K // 8 - 1
        assert set(f.meta[t].tolist()) == ({0x4444} if last else {0xEEEE})
        assert f.nevict[t] == (0 if last else 8)
    # queue order: main tiles pop columns in ascending order; evicted ones follow
    assert f.col_idx[0][8:].tolist() == list(range(8, 16))
    _check(A, f)


def test_all_zero_panel():
    A = np.zeros((256, 64), np.float16)
    A[130, 5] = 1.0                      # panel 1 has one column; panel 0 has none
    f = oracle.reorder(A, P=128)
    assert f.T.tolist() == [0, 1]
    _check(A, f)


@pytest.mark.parametrize("seed", [1, 2])
def test_already_24_needs_no_reorder(seed):
    """a matrix that already satisfies 2:4 'can be directly computed
    without reordering': identity perm, no evictions, T_p = K/16."""
    A = synth.nm24(256, 128, seed)
    f = oracle.reorder(A, P=128)
    assert f.T.tolist() == [8, 8]
    assert int(f.nevict.sum()) == 0
    assert all(f.perm[t].tolist() == list(range(16)) for t in range(len(f.perm)))
    assert np.array_equal(f.col_idx[:8].reshape(-1), np.arange(128))
    _check(A, f)


@pytest.mark.parametrize("V,Mb,K", [(128, 12, 192), (128, 20, 400), (256, 40, 400), (128, 100, 256)])
def test_venom_aligned_needs_no_reorder(V, Mb, K):
    """SURVEY §8f f4 (§4.5): a V:2:Mb matrix with V a multiple of the
    panel height and 4 | Mb is 2:4 inside every block of its compacted columns,
    so CR1 must leave it as it is -- S_p = the 4 selected columns of every
    column block in ascending order, identity permutation on every tile, no
    eviction, T_p = ceil(K_p / 16) -- and the format decodes to A."""
    A = synth.venom(256, K, V, Mb, 31)
    f = oracle.reorder(A, P=128)
    nblk = -(-K // Mb)
    for p in range(len(f.T)):
        blk = A[p * 128:(p + 1) * 128]
        cols = np.flatnonzero(((blk & 0x7FFF) != 0).any(axis=0))
        assert len(cols) == 4 * nblk - (4 - min(4, K - (nblk - 1) * Mb))  # 4 selected per block
        assert f.T[p] == -(-len(cols) // 16)
        toff = f.tile_off
        assert int(f.nevict[toff[p]:toff[p + 1]].sum()) == 0
        for t in range(toff[p], toff[p + 1]):
            n_real = int((f.col_idx[t] >= 0).sum())
            assert f.perm[t][:n_real].tolist() == list(range(n_real))
        got = f.col_idx[toff[p]:toff[p + 1]].reshape(-1)
        assert np.array_equal(got[got >= 0], cols)
    _check(A, f)


@pytest.mark.parametrize("V,Mb", [(32, 12), (64, 20), (32, 100)])
def test_venom_short_vectors_reordered_validly(V, Mb):
    """V:2:Mb with V < P: a 128-row panel spans several V-blocks with different
    column selections, so the union is no longer 2:4 in order and CR1 has real
    work; the format must stay valid, bounded and decode to A."""
    A = synth.venom(256, 400, V, Mb, 32)
    f = oracle.reorder(A, P=128)
    _check(A, f)
    for p in range(len(f.T)):
        blk = A[p * 128:(p + 1) * 128]
        Kp = int(((blk & 0x7FFF) != 0).any(axis=0).sum())
        assert -(-Kp // 16) <= f.T[p] <= Kp // 8 + 1


@pytest.mark.parametrize("M,K,v,s,P,kind,mode", [
    (256, 256, 4, 0.80, 128, "uniform", 0),      # C1
    (256, 256, 4, 0.80, 128, "uniform", 1),
    (200, 160, 8, 0.90, 64, "uniform", 0),       # ragged last panel, P = 64
    (256, 512, 2, 0.70, 128, "skewed", 0),
    (128, 192, 8, 0.50, 128, "uniform", 0),      # residual-heavy regime
    (128, 192, 8, 0.50, 128, "uniform", 1),
    (96, 100, 4, 0.95, 32, "uniform", 0),        # K not a multiple of 16
    (64, 64, 1, 0.0, 64, "uniform", 0),          # fully dense
    (512, 384, 8, 0.90, 256, "uniform", 0),      # 256-row panels (CTA-pair option, R-Q6)
    (600, 256, 4, 0.80, 256, "uniform", 1),      # 256-row panels, ragged, DENSE mode
])
def test_format_valid_and_bounded(M, K, v, s, P, kind, mode):
    A = synth.vector_sparse(M, K, v, s, 17, kind=kind)
    f = oracle.reorder(A, P=P, mode=mode)
    _check(A, f)
    toff = f.tile_off
    for p in range(len(f.T)):
        blk = A[p * P:(p + 1) * P]
        Kp = int(((blk & 0x7FFF) != 0).any(axis=0).sum())
        assert f.T[p] <= Kp // 8 + 1                          # T_p <= floor(K_p/8) + 1
        assert f.T[p] >= -(-Kp // 16)
        ev = f.nevict[toff[p]:toff[p + 1]]
        assert np.all(ev <= 8)
        if mode == 1:
            # DENSE mode: main tiles only (ceil(K_p/16)); evictions land in D_p tiles
            assert f.T[p] == -(-Kp // 16)
            assert f.D[p] == -(-int(ev.sum()) // 16)
        kinds = f.kind[toff[p]:toff[p + 1]]
        nmain = -(-Kp // 16)
        assert kinds.tolist() == [0] * min(nmain, int(f.T[p])) + [1] * (int(f.T[p]) - nmain)
    assert check.format_bytes(f.T, P, f.D if mode == 1 else None) == \
        (18 * P + 64) * int(f.T.sum()) + ((32 * P + 64) * int(f.D.sum()) if mode == 1 else 0)


def test_panel_range_equals_full_run():
    A = synth.vector_sparse(512, 256, 4, 0.8, 3)
    full = oracle.reorder(A, P=128)
    part = oracle.reorder(A, P=128, panels=(1, 3))
    t0, t1 = full.tile_off[1], full.tile_off[3]
    assert np.array_equal(part.T, full.T[1:3])
    assert np.array_equal(part.vals, full.vals[t0:t1])
    assert np.array_equal(part.meta, full.meta[t0:t1])
    assert np.array_equal(part.col_idx, full.col_idx[t0:t1])
    _check(A, part)


def test_negative_zero_is_zero():
    """R-Q3: -0 entries are zeros (not columns of S_p); stored values are canonical +0."""
    A = np.zeros((8, 32), np.float16)
    A[0, 3] = 1.0
    A[1, 5] = -0.0
    f = oracle.reorder(A, P=8)
    ci = f.col_idx[0]
    assert ci[ci != -1].tolist() == [3]
    _check(A, f)


@pytest.mark.parametrize("corrupt", ["meta", "perm", "drop", "val"])
def test_checker_rejects_corruption(corrupt):
    """O3 catches a wrong metadata bit, a wrong permutation, a dropped column and
    a wrong value -- so a format that passes it is a faithful encoding."""
    A = synth.vector_sparse(128, 128, 4, 0.8, 5)
    f = oracle.reorder(A, P=128)
    g, vals, meta, perm = f.gather.copy(), f.vals.copy(), f.meta.copy(), f.perm.copy()
    if corrupt == "meta":
        r = int(np.argmax((vals[0] != 0).any(axis=1)))
        meta[0, r] ^= 0x4          # move i1 of group 0
    elif corrupt == "perm":
        perm[0, [0, 1]] = perm[0, [1, 0]]
        g = np.take_along_axis(f.col_idx, perm.astype(np.int64), axis=1)
        g[0, [0, 5]] = g[0, [5, 0]]
    elif corrupt == "drop":
        j = int(np.argmax(g[0] != -1))
        g[0, j] = -1
    else:
        t, r, k = np.argwhere(vals != 0)[0]
        vals[t, r, k] ^= 0x0001
    with pytest.raises(AssertionError):
        check.check_format(A, f.P, f.T, g, vals, meta, perm=perm)


def test_expected_surviving_columns_matches_hypergeometric():
    """Generator + compaction against a closed form: with exactly nnz of the
    (M/v)*K vector cells nonzero, a panel column (P/v cells) is all-zero with
    probability C(ncell - P/v, nnz) / C(ncell, nnz) (~ s^(P/v))."""
    from math import comb
    M, K, v, s, P = 64, 64, 8, 0.9, 64
    ncell = (M // v) * K
    nnz = int(round((1 - s) * ncell))
    p_zero = comb(ncell - P // v, nnz) / comb(ncell, nnz)
    ks = []
    for seed in range(300):
        A = synth.vector_sparse(M, K, v, s, seed)
        f = oracle.reorder(A, P=P)
        ks.append(int((f.col_idx[f.col_idx != -1] >= 0).sum()))
    mean = np.mean(ks)
    expect = K * (1 - p_zero)
    sd = np.std(ks) / np.sqrt(len(ks))
    assert abs(mean - expect) < 5 * sd + 0.05
