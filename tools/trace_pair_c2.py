"""Per-CTA timeline of the grouped C2 launch, 128-row vs 256-row panels.  Developer tool."""
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
    pts = synth.c2_points()
    mats = [(synth.vector_sparse(M, K, v, s, 50 + i), synth.dense_b(K, N, 50 + i), v)
            for i, (M, K, v, s, N) in enumerate(pts)]
    B2 = [dev(b) for _, b, _ in mats]
    C2 = [torch.empty((a.shape[0], b.shape[1]), dtype=torch.float16, device="cuda") for a, b, _ in mats]
    kp = int(os.environ.get("KPIECES", "0"))
    for P, nt in [(128, 0), (256, 256)]:
        jig.set_launch_override(tile_n=nt, k_pieces=kp)
        hs = [jig.reorder(dev(a), v, panel_rows=P) for a, _, v in mats]
        for rep in range(3):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            jig.spmm_batched(hs, B2, C2)
            e1.record()
            torch.cuda.synchronize()
        tr = jig.debug_trace()
        report(f"grouped C2 P={P} NT={nt or 'auto'} {jig.last_launch()}", e0.elapsed_time(e1) * 1e3, tr, ghz)
        kb = np.zeros(8 * 6 * 32, np.int64)
        jig.lib().jigsaw_debug_trace(kb.ctypes.data_as(ctypes.c_void_p), -1)
        kb = kb.reshape(8, 6, 32)
        for cta in range(2):
            t0 = tr[cta, 0]
            print(f"  CTA {cta} per k-block (us after entry): AE-issue / B-issue / full-seen / after-cp / after-mma / commit")
            for k in range(0, 32, 4):
                row = [(kb[cta, r, k] - t0) / ghz / 1e3 if kb[cta, r, k] > t0 else float('nan') for r in (0, 1, 2, 4, 5, 3)]
                print("   kb %2d  " % k + "  ".join(f"{x:7.2f}" for x in row))
        for h in hs:
            h.free()


if __name__ == "__main__":
    main()
