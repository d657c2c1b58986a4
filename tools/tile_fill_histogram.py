"""Real (non-PAD) columns per 2:4 tile of CR1 formats at the C2 points (oracle,
first two 128-row panels of every matrix): how many overflow tiles would a
CUDA-core path for nearly empty tiles ever see?  CPU tool."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import synth  # noqa: E402

tot = np.zeros(17, np.int64)
print("M x K v s : tiles, histogram of real columns per tile (0..16), tiles with <= 4 real columns")
for i, (M, K, v, s, N) in enumerate(synth.c2_points()):
    A = synth.vector_sparse(M, K, v, s, synth.SEED_BASE + i)
    f = oracle.reorder(A, P=128, panels=(0, 2))
    real = (f.col_idx != -1).sum(1)
    h = np.bincount(real, minlength=17)
    tot += h
    print(f"{M}x{K} v{v} s{s:.2f}: {len(real)} tiles {h.tolist()} le4={int(h[:5].sum())}")
print("all:", tot.tolist(), "tiles with <= 4 real columns:", int(tot[:5].sum()), "of", int(tot.sum()))
