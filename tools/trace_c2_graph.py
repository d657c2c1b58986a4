"""Per-CTA timeline of the C2 grouped launch exactly as bench.py times it (a CUDA
graph of [event, k_spmm, event] replayed after an L2 flush).  Developer tool."""
import os
import sys

os.environ["JIGSAW_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools.trace_spmm import report  # noqa: E402


def main():
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    flush = torch.empty(bench.FLUSH_BYTES, dtype=torch.uint8, device=dev)
    name = sys.argv[1] if len(sys.argv) > 1 else "c2"
    b = bench.Batch(name, 0, 1, 0, dev, torch, jig)
    b.step(jig)
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True, external=True)
    e1 = torch.cuda.Event(enable_timing=True, external=True)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        e0.record()
        b.step(jig)
        e1.record()
    for _ in range(5):
        flush.zero_()
        g.replay()
        torch.cuda.synchronize()
    report(f"graph-replayed {name} (bench timing) {jig.last_launch()}", e0.elapsed_time(e1) * 1e3,
           jig.debug_trace(), 1.965)


if __name__ == "__main__":
    main()
