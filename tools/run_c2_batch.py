"""Runs the C2 batch (36 matrices) through jigsaw_spmm_batched a few times:
a short, ncu-friendly driver for profiling the grouped k_spmm launch."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402


def main(reps=4, wl="c2"):
    torch.cuda.set_device(0)
    pts = synth.c2_points() if wl == "c2" else synth.c4_points()
    hs, Bs, Cs = [], [], []
    for i, (M, K, v, s, N) in enumerate(pts):
        A = synth.vector_sparse(M, K, v, s, i)
        hs.append(jig.reorder(torch.from_numpy(A.view(np.int16)).cuda().view(torch.float16), v, panel_rows=0))
        Bs.append(torch.from_numpy(synth.dense_b(K, N, i).view(np.int16)).cuda().view(torch.float16))
        Cs.append(torch.empty((M, N), dtype=torch.float16, device="cuda"))
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(reps):
        flush.zero_()
        jig.spmm_batched(hs, Bs, Cs)
    torch.cuda.synchronize()
    print("done")


if __name__ == "__main__":
    main(wl=sys.argv[1] if len(sys.argv) > 1 else "c2")
