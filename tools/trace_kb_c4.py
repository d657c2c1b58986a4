"""Per-k-block timeline (library built with tools/build_dev.sh "JIG_TRACE_KB_ON=1",
loaded through JIGSAW_LIB_AB) of CTAs 0/1 on one C4 matrix: the interval between
successive A/E issues, B issues, stage-full observations and commits shows which
role paces the pipeline.  Developer tool."""
import ctypes
import os
import sys

import numpy as np

os.environ["JIGSAW_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools.trace_spmm import dev  # noqa: E402


def main():
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    M, K, v, s, N = (11008, 4096, 8, 0.9, 2048)
    h = jig.reorder(dev(synth.vector_sparse(M, K, v, s, 50)), v, panel_rows=0)
    B = dev(synth.dense_b(K, N, 50))
    C = torch.empty((M, N), dtype=torch.float16, device="cuda")
    for _ in range(3):
        flush.zero_()
        h.spmm(B, C=C)
    torch.cuda.synchronize()
    tr = jig.debug_trace()
    kb = np.zeros(8 * 6 * 32, np.int64)
    jig.lib().jigsaw_debug_trace(kb.ctypes.data_as(ctypes.c_void_p), -1)
    kb = kb.reshape(8, 6, 32)
    names = ["AE issue", "B issue", "full seen", "commit", "own landed", "after mma"]
    print(f"dbg={os.environ.get('JIGSAW_DBG', '0')}  (cycles after CTA entry; d = mean interval over k-blocks 8..31)")
    for c in range(2):
        t0 = tr[c, 0]
        if c == 1:
            names = ["AE issue", "B issue (w0)", "stage landed", "B issue (last w)", "-", "-"]
        for r, nm in enumerate(names):
            row = [(x - t0) for x in kb[c, r] if x > 0]
            d = np.diff(row[8:]).mean() if len(row) > 10 else float("nan")
            print(f"  cta{c} {nm:10s} d={d:7.0f}  " + " ".join(f"{x:7d}" for x in row[:14]))


if __name__ == "__main__":
    main()
