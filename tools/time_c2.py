"""Median device time of the grouped C2 launch (L2 flushed before each rep), eager
and CUDA-graph, for both panel heights and forced tile widths.  Developer tool."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools.trace_spmm import dev  # noqa: E402


def med(fn, flush, reps=30):
    ts = []
    for _ in range(reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return float(np.median(ts)), float(np.min(ts))


def main():
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    wl = sys.argv[1] if len(sys.argv) > 1 else "c2"
    pts = synth.c2_points() if wl == "c2" else synth.c4_points()
    mats = [(synth.vector_sparse(M, K, v, s, 50 + i), synth.dense_b(K, N, 50 + i), v)
            for i, (M, K, v, s, N) in enumerate(pts)]
    B2 = [dev(b) for _, b, _ in mats]
    C2 = [torch.empty((a.shape[0], b.shape[1]), dtype=torch.float16, device="cuda") for a, b, _ in mats]
    configs = [(128, "", ""), (128, "", "1"), (256, "256", ""), (256, "256", "1"), (256, "128", "")]
    for P, nt, nopieces in configs:
        for k, val in (("JIGSAW_FORCE_NT", nt), ("JIGSAW_NO_PIECES", nopieces)):
            if val:
                os.environ[k] = val
            else:
                os.environ.pop(k, None)
        hs = [jig.reorder(dev(a), v, panel_rows=P) for a, _, v in mats]
        step = lambda: jig.spmm_batched(hs, B2, C2)  # noqa: E731
        step()
        torch.cuda.synchronize()
        eager = med(step, flush)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            step()
        graph = med(g.replay, flush)
        print(f"{wl} P={P} NT={nt or 'auto'} pieces={'off' if nopieces else 'on'}: eager median {eager[0]:.1f} "
              f"(min {eager[1]:.1f}) us, graph median {graph[0]:.1f} (min {graph[1]:.1f}) us", flush=True)
        for h in hs:
            h.free()


if __name__ == "__main__":
    main()
