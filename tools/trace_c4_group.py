"""Per-CTA timeline of the grouped C4 launch (CTA pairs, static LPT schedule):
finish-time spread = load imbalance.  Developer tool."""
import os
import sys

os.environ["JIGSAW_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools.trace_spmm import report, dev  # noqa: E402


def main():
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    wl = sys.argv[1] if len(sys.argv) > 1 else "c4"
    P = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    pts = synth.c4_points() if wl == "c4" else synth.c2_points()
    mats = [(synth.vector_sparse(M, K, v, s, 50 + i), synth.dense_b(K, N, 50 + i), v)
            for i, (M, K, v, s, N) in enumerate(pts)]
    hs = [jig.reorder(dev(a), v, panel_rows=P) for a, _, v in mats]
    B2 = [dev(b) for _, b, _ in mats]
    C2 = [torch.empty((a.shape[0], b.shape[1]), dtype=torch.float16, device="cuda") for a, b, _ in mats]
    for rep in range(3):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        jig.spmm_batched(hs, B2, C2)
        e1.record()
        torch.cuda.synchronize()
    report(f"grouped {wl} P={P}", e0.elapsed_time(e1) * 1e3, jig.debug_trace(), 1.965)


if __name__ == "__main__":
    main()
