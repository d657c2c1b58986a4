"""Single-product latency: every C2 point as ONE jigsaw_spmm call and ONE cuBLAS
call (torch.matmul on the dense fp16 A), L2 flushed before each.  Run it under
`ncu --metrics gpu__time_duration.sum` for kernel-only durations; without ncu it
prints the bench-style event times (graph replay between two events).
Developer tool."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x).view(np.int16)).cuda().view(torch.float16)


def main():
    torch.cuda.set_device(0)
    reps = int(os.environ.get("REPS", "3"))
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    pts = synth.c2_points()
    sel = os.environ.get("POINTS")
    if sel:
        pts = [pts[int(i)] for i in sel.split(",")]
    for i, (M, K, v, s, N) in enumerate(pts):
        A = synth.vector_sparse(M, K, v, s, 50 + i)
        dA = dev(A)
        h = jig.reorder(dA, v)
        B = dev(synth.dense_b(K, N, 50 + i))
        C = torch.empty((M, N), dtype=torch.float16, device="cuda")
        C2 = torch.empty_like(C)
        tj, tc = [], []
        for _ in range(reps):
            for fn, acc in ((lambda: h.spmm(B, C=C), tj), (lambda: torch.matmul(dA, B, out=C2), tc)):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                fn()
                e1.record()
                e1.synchronize()
                acc.append(e0.elapsed_time(e1) * 1e3)
        info = h.info()
        print(f"{M}x{K} v{v} s{s} N{N} tiles={info.get('ntiles')} jig {np.median(tj):.2f} us  cublas {np.median(tc):.2f} us",
              flush=True)
        h.free()


if __name__ == "__main__":
    main()
