"""Single-product latency: every C2 point as ONE jigsaw_spmm call and ONE cuBLAS
call (torch.matmul on the dense fp16 A), L2 flushed before each.  Two clocks:
  event  -- events around one graph replay holding one call (bench-style; this
            box's event clock moves in ~2.05 us steps);
  graph  -- a graph of R x (flush, call) minus a graph of R x (flush), / R: the
            call's device time in a stream of back-to-back kernels, resolved to
            ~0.1 us.
Developer tool (POINTS=i,j,... selects C2 points, REPS the repetitions)."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x).view(np.int16)).cuda().view(torch.float16)


def graph_of(fn, R, flush):
    fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(R):
            flush.zero_()
            if fn is not None:
                fn()
    return g


def time_graph(g, reps):
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return float(np.median(ts))


def main():
    torch.cuda.set_device(0)
    reps = int(os.environ.get("REPS", "3"))
    R = 16
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    pts = synth.c2_points()
    sel = os.environ.get("POINTS")
    if sel:
        pts = [pts[int(i)] for i in sel.split(",")]
    g0 = graph_of(lambda: None, R, flush)
    for i, (M, K, v, s, N) in enumerate(pts):
        A = synth.vector_sparse(M, K, v, s, 50 + i)
        dA = dev(A)
        h = jig.reorder(dA, v)
        B = dev(synth.dense_b(K, N, 50 + i))
        C = torch.empty((M, N), dtype=torch.float16, device="cuda")
        C2 = torch.empty_like(C)
        fj = lambda: h.spmm(B, C=C)  # noqa: E731
        fc = lambda: torch.matmul(dA, B, out=C2)  # noqa: E731
        tj, tc = [], []
        for _ in range(reps):
            for fn, acc in ((fj, tj), (fc, tc)):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                fn()
                e1.record()
                e1.synchronize()
                acc.append(e0.elapsed_time(e1) * 1e3)
        t0 = time_graph(g0, 5)
        gj = (time_graph(graph_of(fj, R, flush), 5) - t0) / R
        gc = (time_graph(graph_of(fc, R, flush), 5) - t0) / R
        info = h.info()
        print(f"{M}x{K} v{v} s{s} N{N} tiles={info.get('ntiles')}  event: jig {np.median(tj):.2f} cublas {np.median(tc):.2f} us"
              f"  graph: jig {gj:.2f} cublas {gc:.2f} us  speedup {gc / gj:.2f}", flush=True)
        h.free()


if __name__ == "__main__":
    main()
