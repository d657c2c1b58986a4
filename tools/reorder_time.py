"""GPU reorder (R1-R5) device time per matrix (jigsaw_get_info.reorder_ms) and
wall time, C2 and C4 shapes.  Developer tool."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools.trace_spmm import dev  # noqa: E402


def main():
    torch.cuda.set_device(0)
    pts = [p for p in synth.c2_points() if p[0] == 512] + synth.c4_points()
    for i, (M, K, v, s, N) in enumerate(pts):
        A = dev(synth.vector_sparse(M, K, v, s, 90 + i))
        torch.cuda.synchronize()
        t = time.perf_counter()
        h = jig.reorder(A, v, panel_rows=0)
        w = (time.perf_counter() - t) * 1e3
        inf = h.info()
        print(f"{M}x{K} v{v} s{s}: reorder device {inf['reorder_ms']:8.2f} ms wall {w:8.2f} ms  tiles {inf['ntiles']}"
              f" evictions {inf['evictions']} P {inf['panel_rows']}", flush=True)
        h.free()


if __name__ == "__main__":
    main()
