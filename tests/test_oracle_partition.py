"""Pins for the tile search of oracle O2: Alg. 1 + reorder retry (PAPER.md
P:146-190) as fixed by readings R-Q8 (lexicographically first cover) and R-Q11
(least-frequent eviction, ties to the smallest slot).

Pinned against: exhaustive enumeration of all 2,627,625 partitions of 16
columns into four 4-column groups; the P = 1 closed form; the Fig. 6 worked
example; the hand-derived eviction case of SURVEY §8c."""
import itertools
import json
import os

import numpy as np
import pytest

import oracle


def _all_partitions_lex():
    """Every partition of {0..15} into 4 groups of 4, groups sorted, ordered by
    their minimum, listed in lexicographic order of (g0, g1, g2, g3)."""
    out = []

    def rec(rest, acc):
        if not rest:
            out.append(acc)
            return
        lo = rest[0]
        for tri in itertools.combinations(rest[1:], 3):
            g = (lo,) + tri
            rec([x for x in rest if x not in g], acc + [g])

    rec(list(range(16)), [])
    return out


@pytest.fixture(scope="module")
def partitions():
    parts = _all_partitions_lex()
    assert len(parts) == 2627625
    masks = np.array([[sum(1 << j for j in g) for g in p] for p in parts], dtype=np.int64)
    return parts, masks


def _compat_table(m, Z=2):
    """compat[mask] for every 4-subset: no row has more than Z nonzeros (direct row count)."""
    rows = max(x.bit_length() for x in m) if any(m) else 1
    tab = np.zeros(1 << 16, dtype=bool)
    for g in itertools.combinations(range(16), 4):
        cnt = [sum((m[j] >> r) & 1 for j in g) for r in range(rows)]
        tab[sum(1 << j for j in g)] = max(cnt, default=0) <= Z
    return tab


def test_partition_matches_exhaustive_enumeration(partitions):
    parts, masks = partitions
    rng = np.random.default_rng(2024)
    n_ok = n_fail = 0
    for trial in range(40):
        P = int(rng.choice([1, 3, 8, 16, 40, 64, 128, 200, 256]))
        dens = float(rng.uniform(0.1, 0.6))
        m = [int(sum(1 << r for r in range(P) if rng.random() < dens)) for _ in range(16)]
        m = [x if x else 1 << int(rng.integers(P)) for x in m]      # real columns are nonzero
        tab = _compat_table(m)
        valid = tab[masks].all(axis=1)
        perm, cols, ev = oracle.tile_reorder(m, list(range(16)))
        if valid.any():
            n_ok += 1
            first = parts[int(np.argmax(valid))]
            assert ev == [] and perm == [j for g in first for j in g]
        else:
            n_fail += 1
            assert len(ev) >= 1
    assert n_ok >= 5 and n_fail >= 5


def test_single_row_closed_form():
    """P = 1: a cover exists iff at most 8 of the 16 columns are nonzero (every
    group may hold at most 2 of the row's nonzeros).  Exhaustive over 2^16."""
    for x in range(1 << 16):
        real = [j for j in range(16) if (x >> j) & 1]
        cols = [j if (x >> j) & 1 else -1 for j in range(16)]
        masks = [1 if (x >> j) & 1 else 0 for j in range(16)]
        _, _, ev = oracle.tile_reorder(masks, cols)
        if len(real) <= 8:
            assert ev == []
        else:
            # each eviction removes one nonzero; it stops exactly at 8
            assert len(ev) == len(real) - 8


def test_fig6_worked_example(golden_dir):
    """columns 7, 8, 10, 11 form one MMA_TILE (1:2 pattern, 4 wide);
    {7,8} conflict (e1, f1); the reorder pairs 7 with 10 and 8 with 11."""
    g = json.load(open(os.path.join(golden_dir, "fig6_format.json")))
    c7, c8, c10, c11 = g["mma_tile_columns"]
    # rows: 0 -> e1 (col 7) and f1 (col 8); 1 -> cols 10, 11; 2 -> col 7 alone
    m = {c7: 0b101, c8: 0b001, c10: 0b010, c11: 0b010}
    cols = [c7, c8, c10, c11]
    perm, _, ev = oracle.tile_reorder([m[c] for c in cols], cols, W=4, G=2, Z=1)
    assert ev == []
    order = [cols[j] for j in perm]
    groups = [sorted(order[0:2]), sorted(order[2:4])]
    assert groups == g["expected_groups"]
    # same groups as the paper's order 7,10 | 11,8 (R-Q10)
    po = g["paper_order"]
    assert sorted(map(sorted, [po[0:2], po[2:4]])) == sorted(groups)


def test_fig6_block_tile_compaction(golden_dir):
    """all-zero columns 3,5,6,9 of a 12-column BLOCK_TILE go to the end;
    col_idx_array keeps the remaining columns (ascending, R-Q4)."""
    g = json.load(open(os.path.join(golden_dir, "fig6_format.json")))
    K = g["block_tile_columns"]
    A = np.zeros((4, K), np.float16)
    for c in range(K):
        if c not in g["zero_columns"]:
            A[c % 4, c] = 1.0
    f = oracle.reorder(A, P=4)
    assert f.T.tolist() == [1]
    ci = f.col_idx[0]
    assert ci[ci != -1].tolist() == g["expected_col_idx"]


def test_eviction_hand_derived(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "eviction_p9.json")))
    A = np.ones((8, 9), np.float16)
    f = oracle.reorder(A, P=8)
    assert f.T.tolist() == [g["T_p"]]
    assert f.col_idx[0].tolist() == g["tile0_col_idx"]
    assert f.perm[0].tolist() == g["tile0_perm"]
    assert f.col_idx[1].tolist() == g["tile1_col_idx"]
    assert f.perm[1].tolist() == g["tile1_perm"]
    assert set(f.meta[0].tolist()) == {int(g["tile0_meta"], 16)}
    assert set(f.meta[1].tolist()) == {int(g["tile1_meta"], 16)}
    assert f.nevict.tolist() == [1, 0]
    assert f.kind.tolist() == [0, 1]


def test_eviction_frequency_rule():
    """the evicted column is the real column contained in the fewest
    compatible 4-groups (counted here by brute force), ties to the smallest slot."""
    rng = np.random.default_rng(7)
    checked = 0
    for _ in range(60):
        P = 16
        m = [int(sum(1 << r for r in range(P) if rng.random() < 0.45)) or 1 for _ in range(16)]
        tab = _compat_table(m)
        freq = [sum(tab[sum(1 << j for j in g)] for g in itertools.combinations(range(16), 4)
                    if s in g) for s in range(16)]
        perm, cols, ev = oracle.tile_reorder(m, list(range(16)))
        if ev:   # (whether a cover exists is pinned by the exhaustive test above)
            assert ev[0] == int(np.argmin(freq))
            checked += 1
    assert checked >= 10
