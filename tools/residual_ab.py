"""SPTC vs DENSE residual mode on C4-shaped matrices at low sparsity:
single products, L2 flushed, graph-difference timing.  Developer tool."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools.trace_spmm import dev  # noqa: E402
from tools.single_c2 import graph_of, time_graph  # noqa: E402


def main():
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    R = 4
    g0 = graph_of(lambda: None, R, flush)
    for (M, K, v, s, N) in [(4096, 4096, 8, 0.5, 2048), (4096, 4096, 8, 0.7, 2048), (11008, 4096, 8, 0.5, 2048),
                            (4096, 4096, 4, 0.7, 2048), (512, 2048, 4, 0.5, 256)]:
        A = dev(synth.vector_sparse(M, K, v, s, 7))
        B = dev(synth.dense_b(K, N, 7))
        C = torch.empty((M, N), dtype=torch.float16, device="cuda")
        Cd = torch.empty_like(C)
        t0 = time_graph(g0, 5)
        tc = (time_graph(graph_of(lambda: torch.matmul(A, B, out=Cd), R, flush), 5) - t0) / R
        row = f"{M}x{K} v{v} s{s} N{N}: cuBLAS {tc:7.1f} us"
        for P in (128, 256):
            for mode in (0, 1):
                h = jig.reorder(A, v, panel_rows=P, residual_mode=mode)
                info = h.info()
                tj = (time_graph(graph_of(lambda: h.spmm(B, C=C), R, flush), 5) - t0) / R
                row += f" | P{P} {'SPTC' if mode == 0 else 'DENSE'} {tj:7.1f} us (tiles {info['ntiles']} dense {info['ndtiles']})"
                h.free()
        print(row, flush=True)


if __name__ == "__main__":
    main()
