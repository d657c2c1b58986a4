"""Per-CTA and per-k-block timeline of k_spmm for one large product, 128-row
panels vs 256-row panels (CTA pairs) at N tiles of 128 / 256.  Developer tool."""
import ctypes
import os
import sys

import numpy as np

os.environ["JIGSAW_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools.trace_spmm import report, dev  # noqa: E402


def main():
    torch.cuda.set_device(0)
    ghz = 1.965
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    M, K, N, v, s = 4096, 4096, 2048, 8, 0.9
    A = synth.vector_sparse(M, K, v, s, 3)
    B = dev(synth.dense_b(K, N, 3))
    C = torch.empty((M, N), dtype=torch.float16, device="cuda")
    for P, nt, dbg in [(256, "256", "0"), (128, "128", "0")]:
        os.environ["JIGSAW_FORCE_NT"] = nt
        os.environ["JIGSAW_DBG"] = dbg
        h = jig.reorder(dev(A), v, panel_rows=P)
        for rep in range(3):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            h.spmm(B, C=C)
            e1.record()
            torch.cuda.synchronize()
        tr = jig.debug_trace()
        report(f"dbg={dbg} P={P} NT={nt} {M}x{K} v{v} s{s} N{N}", e0.elapsed_time(e1) * 1e3, tr, ghz)
        kb = np.zeros(8 * 6 * 32, np.int64)
        jig.lib().jigsaw_debug_trace(kb.ctypes.data_as(ctypes.c_void_p), -1)
        kb = kb.reshape(8, 6, 32)
        for cta in range(1):
            t0 = tr[cta, 0]
            print(f"  CTA {cta} per k-block (us after entry): AE-issue / B-issue / full-seen / after-cp / after-mma / commit")
            for k in range(8, 16, 2):
                row = [(kb[cta, r, k] - t0) / ghz / 1e3 if kb[cta, r, k] > t0 else float('nan') for r in (0, 1, 2, 4, 5, 3)]
                print("   kb %2d  " % k + "  ".join(f"{x:7.2f}" for x in row))
        h.free()


if __name__ == "__main__":
    main()
