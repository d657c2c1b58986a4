"""O3 -- independent checker / decoder of a reorder-aware format (numpy).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  It never calls the CR1
reorder (O2): it only checks that a given format is a VALID encoding of A,
whatever produced it (the oracle, or the GPU library via jigsaw_export_format).

Checks:
  * bijection   -- per panel the non-PAD gather entries are exactly the columns
                   with any nonzero in the panel, each once;
  * perm        -- every perm[t] is a permutation of 0..15 (when given);
  * 2:4         -- per row/tile/group at most 2 nonzeros among the 4 mapped
                   columns, every one of them selected by the metadata;
  * metadata    -- i0 < i1 in every nibble;
  * PAD         -- values at PAD positions are +0;
  * CUDA-core   -- (f3, R-Q28) entries (row, column, value) of a panel are in
    entries        strictly increasing (row, column) order, inside the panel,
                   nonzero; their columns are disjoint from the tiles' columns;
  * decode      -- decode(format) == canon(A) bitwise (canon: -0 -> +0, R-Q3).
"""
from __future__ import annotations

import numpy as np

PAD = -1


def canon(A: np.ndarray) -> np.ndarray:
    """fp16 bits with -0 mapped to +0 (R-Q3)."""
    A = np.asarray(A).view(np.uint16).copy()
    A[(A & 0x7FFF) == 0] = 0
    return A


def _nz(x):
    return (x & 0x7FFF) != 0


def decode(M, K, P, T, gather, vals, meta, D=None, rcol=None, dvals=None, cc=None):
    """Rebuild the M x K fp16-bit matrix from the format.
    ``cc`` = (eoff, row, col, val): CUDA-core entries per panel (f3)."""
    out = np.zeros((M, K), np.uint16)
    npan = len(T)
    toff = np.concatenate([[0], np.cumsum(T)]).astype(np.int64)
    doff = np.concatenate([[0], np.cumsum(D)]).astype(np.int64) if D is not None else None
    for p in range(npan):
        r0 = p * P
        nr = min(P, M - r0)
        for t in range(toff[p], toff[p + 1]):
            g = gather[t]
            for q in range(4):
                for k in range(2):
                    pos = (meta[t, :nr].astype(np.int64) >> (4 * q + 2 * k)) & 3
                    col = g[4 * q + pos]
                    v = vals[t, :nr, 2 * q + k]
                    ok = col != PAD
                    rr = np.arange(nr)[ok]
                    out[r0 + rr, col[ok]] = v[ok]
        if doff is not None:
            for d in range(doff[p], doff[p + 1]):
                for j in range(16):
                    c = rcol[d, j]
                    if c != PAD:
                        out[r0:r0 + nr, c] = dvals[d, :nr, j]
        if cc is not None:
            eoff, crow, ccol, cval = cc
            e = slice(int(eoff[p]), int(eoff[p + 1]))
            out[r0 + crow[e].astype(np.int64), ccol[e]] = cval[e]
    return out


def format_bytes(T, P, D=None):
    """Format size closed form (R-Q19, our layout): per 2:4 tile 16 B values +
    2 B metadata per row plus 64 B gather; per dense tile 32 B per row + 64 B."""
    T = np.asarray(T)
    nb = int((16 * P + 2 * P + 64) * T.sum())
    if D is not None:
        nb += int((32 * P + 64) * np.asarray(D).sum())
    return nb


def check_format(A, P, T, gather, vals, meta, perm=None, D=None, rcol=None, dvals=None,
                 panels=None, cc=None):
    """Raise AssertionError if the format is not a valid encoding of A.

    ``panels``: range of panel indices the format covers (default: all).
    ``cc`` = (eoff, row, col, val): CUDA-core entries per panel (f3)."""
    A = np.asarray(A).view(np.uint16)
    M, K = A.shape
    npan_all = (M + P - 1) // P
    panels = range(npan_all) if panels is None else panels
    T = np.asarray(T)
    assert len(T) == len(panels)
    toff = np.concatenate([[0], np.cumsum(T)]).astype(np.int64)
    doff = np.concatenate([[0], np.cumsum(D)]).astype(np.int64) if D is not None else None
    if perm is not None:
        for t in range(len(perm)):
            assert sorted(perm[t].tolist()) == list(range(16)), f"tile {t}: perm not a permutation"
    for i, p in enumerate(panels):
        r0 = p * P
        nr = min(P, M - r0)
        blk = A[r0:r0 + nr]
        S = np.nonzero(_nz(blk).any(axis=0))[0]
        g = gather[toff[i]:toff[i + 1]].reshape(-1)
        used = g[g != PAD]
        if doff is not None:
            rc = rcol[doff[i]:doff[i + 1]].reshape(-1)
            used = np.concatenate([used, rc[rc != PAD]])
        if cc is not None:
            eoff, crow, ccol, cval = cc
            e = slice(int(eoff[i]), int(eoff[i + 1]))
            er, ec, ev = crow[e].astype(np.int64), ccol[e].astype(np.int64), cval[e]
            assert np.all((er >= 0) & (er < nr)), f"panel {p}: CUDA-core entry outside the panel"
            assert np.all(_nz(ev)), f"panel {p}: CUDA-core entry holds a zero"
            key = er * (K + 1) + ec
            assert np.all(np.diff(key) > 0), f"panel {p}: CUDA-core entries not in (row, column) order"
            used = np.concatenate([used, np.unique(ec)])
        assert len(used) == len(np.unique(used)), f"panel {p}: a column appears twice"
        assert np.array_equal(np.sort(used), S), f"panel {p}: gather is not a bijection onto S_p"
        for t in range(toff[i], toff[i + 1]):
            mt = meta[t].astype(np.int64)
            for q in range(4):
                nib = (mt >> (4 * q)) & 0xF
                i0, i1 = nib & 3, nib >> 2
                assert np.all(i0 < i1), f"tile {t} group {q}: metadata not ascending"
                cols = gather[t, 4 * q:4 * q + 4]
                for pos in range(4):
                    c = cols[pos]
                    sel = (i0 == pos) | (i1 == pos)
                    if c == PAD:
                        # PAD positions carry +0 values
                        for k, ik in ((0, i0), (1, i1)):
                            hit = ik == pos
                            assert np.all(vals[t, hit, 2 * q + k] == 0), f"tile {t}: nonzero at PAD"
                        continue
                    colnz = _nz(blk[:, c])
                    assert np.all(sel[:nr] | ~colnz), f"tile {t} group {q}: a nonzero not selected"
    dec = decode(M, K, P, np.asarray(T), gather, vals, meta,
                 D=D, rcol=rcol, dvals=dvals, cc=cc) if panels == range(npan_all) else None
    if dec is not None:
        assert np.array_equal(dec, canon(A)), "decode(format) != canon(A)"
    else:
        # partial panel range: decode only those rows
        for i, p in enumerate(panels):
            r0 = p * P
            nr = min(P, M - r0)
            sub_T = T[i:i + 1]
            sl = slice(toff[i], toff[i + 1])
            dsl = slice(doff[i], doff[i + 1]) if doff is not None else None
            sub_cc = None
            if cc is not None:
                eoff, crow, ccol, cval = cc
                e = slice(int(eoff[i]), int(eoff[i + 1]))
                sub_cc = (np.array([0, e.stop - e.start]), crow[e], ccol[e], cval[e])
            d = decode(nr, K, P, sub_T, gather[sl], vals[sl], meta[sl],
                       D=None if D is None else np.asarray(D)[i:i + 1],
                       rcol=None if rcol is None else rcol[dsl],
                       dvals=None if dvals is None else dvals[dsl], cc=sub_cc)
            assert np.array_equal(d, canon(A[r0:r0 + nr])), f"panel {p}: decode != canon(A)"
    return True
