"""Cold (L2 flushed) vs warm (immediately repeated) timeline of single small
products: separates first-touch latency (code, parameters, data from DRAM)
from the kernel's own critical path.  Developer tool."""
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
    pts = [(512, 2048, 4, 0.9, 256), (2048, 512, 4, 0.9, 256), (512, 2048, 8, 0.98, 256)]
    for i, (M, K, v, s, N) in enumerate(pts):
        h = jig.reorder(dev(synth.vector_sparse(M, K, v, s, i)), v)
        B = dev(synth.dense_b(K, N, i))
        C = torch.empty((M, N), dtype=torch.float16, device="cuda")
        for mode in ("cold", "warm", "warm-B-only-flushed"):
            for rep in range(3):
                if mode == "cold":
                    flush.zero_()
                elif mode == "warm":
                    h.spmm(B, C=C)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                h.spmm(B, C=C)
                e1.record()
                torch.cuda.synchronize()
            if mode == "warm-B-only-flushed":
                continue
            tr = jig.debug_trace()
            report(f"{mode} {M}x{K} v{v} s{s} N{N}", e0.elapsed_time(e1) * 1e3, tr, ghz)
            if os.environ.get("KB"):  # per-k-block timeline (library built with JIG_TRACE_KB_ON=1)
                import ctypes
                kb = np.zeros(8 * 6 * 32, np.int64)
                jig.lib().jigsaw_debug_trace(kb.ctypes.data_as(ctypes.c_void_p), -1)
                kb = kb.reshape(8, 6, 32)
                names = ["AE issue", "B issue", "full seen", "commit", "after cp", "after mma"]
                for c in range(2):
                    t0 = tr[c, 0]
                    for r, nm in enumerate(names):
                        row = [(x - t0) / ghz / 1e3 for x in kb[c, r] if x > 0]
                        print(f"   cta{c} {nm:10s} " + " ".join(f"{x:6.2f}" for x in row[:12]))


if __name__ == "__main__":
    main()
