"""Synthetic analogue of the paper's Fig. 11:
how often the multi-granularity reorder succeeds ("2:4 while keeping K no bigger
than the original", R-Q13) and how much the retry inflates the tile count, vs
vector width v and sparsity s, at the B200 panel height P = 128 -- measured with
the GPU builder (jigsaw_reorder), together with its device time.

  python tools/reorder_study.py > profiles/r01_reorder_study.md
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402


def main():
    torch.cuda.set_device(0)
    shapes = [(512, 2048), (2048, 512), (512, 512), (256, 2304), (4096, 4096)]
    print("# Reorder study (GPU builder, P = 128, uniform random vector pruning, 3 seeds)\n")
    print("success = fraction of panels with 16*T_p <= 16*ceil(K/16) (R-Q13); inflation = "
          "tiles / sum ceil(K_p/16); evict/tile = evictions per tile; DENSE: residual tiles per "
          "panel in DENSE mode; ms = device time of jigsaw_reorder (SPTC)\n")
    print("| M x K | v | s | K_p/K | success | inflation | evict/tile | DENSE tiles/panel | reorder ms |")
    print("|---|---|---|---|---|---|---|---|---|")
    for (M, K) in shapes:
        for v in (2, 4, 8):
            for s in (0.5, 0.7, 0.8, 0.9, 0.95, 0.98):
                succ, infl, evt, kpk, dtp, ms = [], [], [], [], [], []
                for seed in range(3):
                    A = synth.vector_sparse(M, K, v, s, 1000 + seed)
                    dA = torch.from_numpy(A.view(np.int16)).cuda().view(torch.float16)
                    h = jig.reorder(dA, v)
                    inf = h.info()
                    g = h.export()
                    T = g["T"]
                    npan = len(T)
                    kp = inf["kp_total"]
                    main = sum(-(-int(x) // 16) for x in
                               [((A[p * 128:(p + 1) * 128] & 0x7FFF) != 0).any(axis=0).sum()
                                for p in range(npan)])
                    succ.append(float(np.mean(16 * T <= 16 * -(-K // 16))))
                    infl.append(inf["ntiles"] / max(1, main))
                    evt.append(inf["evictions"] / max(1, inf["ntiles"]))
                    kpk.append(kp / (npan * K))
                    ms.append(inf["reorder_ms"])
                    hd = jig.reorder(dA, v, residual_mode=1)
                    dtp.append(hd.info()["ndtiles"] / npan)
                    h.free()
                    hd.free()
                print(f"| {M}x{K} | {v} | {s:.2f} | {np.mean(kpk):.3f} | {np.mean(succ):.2f} | "
                      f"{np.mean(infl):.2f} | {np.mean(evt):.2f} | {np.mean(dtp):.1f} | {np.median(ms):.2f} |",
                      flush=True)


if __name__ == "__main__":
    main()
