"""Synthetic analogue of the paper's Fig. 11 vs panel height: for
BLOCK_TILE / panel heights P = 16, 32, 64 (the paper's sizes), 128 and 256
(the B200 kernel's one-CTA and CTA-pair tcgen05 M), how many columns survive the
panel compaction, how often the multi-granularity reorder succeeds (R-Q13), how
much the retry inflates the tile count, and the resulting executed MMA work as a
fraction of the dense GEMM -- all measured with the GPU builder (jigsaw_reorder).

  python tools/panel_study.py > profiles/r01_panel_study.md
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
    shapes = [(512, 2048), (2048, 512), (4096, 4096)]
    Ps = [16, 32, 64, 128, 256]
    print("# Panel-height study (GPU builder, uniform random vector pruning, 2 seeds)\n")
    print("K_p/K = surviving columns per panel; success = panels with 16*T_p <= 16*ceil(K/16) (R-Q13); "
          "infl = tiles / sum ceil(K_p/16); work = executed 2:4 MMA work / dense GEMM work "
          "(= sum_p 8 * P * T_p / (M*K)); ms = jigsaw_reorder device time.\n")
    hdr = "| M x K | v | s | " + " | ".join(f"P={P} K_p/K, succ, infl, work, ms" for P in Ps) + " |"
    print(hdr)
    print("|" + "---|" * (3 + len(Ps)))
    for (M, K) in shapes:
        for v in (2, 4, 8):
            for s in (0.5, 0.7, 0.8, 0.9, 0.95, 0.98):
                cells = []
                for P in Ps:
                    kpk, succ, infl, work, ms = [], [], [], [], []
                    for seed in range(2):
                        A = synth.vector_sparse(M, K, v, s, 2000 + seed)
                        dA = torch.from_numpy(A.view(np.int16)).cuda().view(torch.float16)
                        h = jig.reorder(dA, v, panel_rows=P)
                        inf = h.info()
                        T = h.export()["T"] if P < 128 or M * K <= 4096 * 4096 else None
                        npan = inf["npanels"]
                        kp = inf["kp_total"]
                        kpk.append(kp / (npan * K))
                        if T is not None:
                            succ.append(float(np.mean(16 * T <= 16 * -(-K // 16))))
                        main = inf["ntiles"] - inf["overflow_tiles"]
                        infl.append(inf["ntiles"] / max(1, main))
                        work.append(8.0 * P * inf["ntiles"] / (M * K))
                        ms.append(inf["reorder_ms"])
                        h.free()
                    cells.append(f"{np.mean(kpk):.2f}, {np.mean(succ) if succ else float('nan'):.2f}, "
                                 f"{np.mean(infl):.2f}, {np.mean(work):.2f}, {np.median(ms):.1f}")
                print(f"| {M}x{K} | {v} | {s:.2f} | " + " | ".join(cells) + " |", flush=True)


if __name__ == "__main__":
    main()
