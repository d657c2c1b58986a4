"""C4-shaped single products, warm (back-to-back, inputs L2-resident where they
fit) vs cold (256 MB L2 flush before each call): is the mainloop bound by the
SM's L2 ingest or by DRAM misses?  Prints us, effective TF/s and SM cycles per
k-block per CTA.  Developer tool."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools.trace_spmm import dev  # noqa: E402


def med(fn, flush, reps=20):
    ts = []
    for _ in range(reps):
        if flush is not None:
            flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return float(np.median(ts))


def main():
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    pts = [(4096, 4096, 8, 0.9, 2048), (4096, 4096, 8, 0.7, 2048), (11008, 4096, 8, 0.9, 2048),
           (4096, 4096, 8, 0.9, 512)]
    for i, (M, K, v, s, N) in enumerate(pts):
        A = synth.vector_sparse(M, K, v, s, 50 + i)
        B = dev(synth.dense_b(K, N, 50 + i))
        C = torch.empty((M, N), dtype=torch.float16, device="cuda")
        dA = dev(A)
        for P in (256, 128):
            h = jig.reorder(dA, v, panel_rows=P)
            info = h.info()
            f = lambda: h.spmm(B, C=C)  # noqa: E731
            f()
            torch.cuda.synchronize()
            tw, tc = med(f, None), med(f, flush)
            Cd = torch.empty_like(C)
            g = lambda: torch.matmul(dA, B, out=Cd)  # noqa: E731
            cw, cc = med(g, None), med(g, flush)
            # k-blocks per CTA: sparse k-steps / 4 per panel x N tiles of 256, over the CTAs
            # (P = 256: a pair per panel, each CTA of the pair ingests its half)
            units_per_cta = info["nksteps"] / 4 * (N / 256) / (74 if P == 256 else 148)
            fl = 2 * M * N * K
            print(f"{M}x{K} v{v} s{s} N{N} P{P}: warm {tw:7.1f} us ({fl / tw / 1e6:6.0f} TF/s)  cold {tc:7.1f} us"
                  f"  | cuBLAS warm {cw:7.1f} cold {cc:7.1f} us  | kblocks/CTA {units_per_cta:6.1f}"
                  f"  cyc/kblock warm {tw * 1965 / max(units_per_cta, 1):6.0f}", flush=True)


if __name__ == "__main__":
    main()
