"""What the bench's step timing (events recorded as graph nodes around the step,
L2 flushed before) adds around a kernel: empty step, a tiny torch kernel, single
jigsaw products (small parameter block), the grouped C2 / C4 launches (31 KB
parameter block) -- event time vs the kernel's own CTA span.  Developer tool."""
import json
import os
import sys

os.environ["JIGSAW_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402


def timed(fn, flush, reps=20, pre=None):
    fn()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True, external=True)
    e1 = torch.cuda.Event(enable_timing=True, external=True)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        e0.record()
        fn()
        e1.record()
    ts = []
    for _ in range(reps):
        flush.zero_()
        if pre is not None:
            pre()
        g.replay()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return float(np.median(ts))


def span():
    tr = jig.debug_trace()
    return float((tr[:, 13].max() - tr[:, 15].min()) / 1e3) if len(tr) else float("nan")


def main():
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    flush = torch.empty(bench.FLUSH_BYTES, dtype=torch.uint8, device=dev)
    x = torch.zeros(1024, device=dev)
    print(json.dumps({"case": "empty", "event_us": timed(lambda: None, flush)}))
    print(json.dumps({"case": "torch add_ (1k floats)", "event_us": timed(lambda: x.add_(1), flush)}))
    b = bench.Batch("c2", 0, 1, 0, dev, torch, jig)
    for i in (0, 30):
        h, B, C = b.hs[i], b.dB[i], b.dC[i]
        us = timed(lambda: h.spmm(B, C), flush)
        print(json.dumps({"case": f"single {b.points[i]}", "event_us": us, "cta_span_us": span(),
                          "launch": jig.last_launch()}))
    for n in (1, 4, 36):
        us = timed(lambda: jig.spmm_batched(b.hs[:n], b.dB[:n], b.dC[:n]), flush)
        print(json.dumps({"case": f"grouped c2 first {n}", "event_us": us, "cta_span_us": span(),
                          "launch": jig.last_launch()}))
    # the same, with a small big-shared-memory kernel (a jigsaw product of a
    # 128 x 64 matrix, unrelated data) between the flush and the timed graph
    import synth
    a = torch.from_numpy(synth.vector_sparse(128, 64, 4, 0.8, 9).view(np.int16)).to(dev).view(torch.float16)
    hs = jig.reorder(a, 4)
    bs = torch.from_numpy(synth.dense_b(64, 64, 9).view(np.int16)).to(dev).view(torch.float16)
    cs = torch.empty((128, 64), dtype=torch.float16, device=dev)
    pre = lambda: hs.spmm(bs, cs)
    for n in (1, 36):
        us = timed(lambda: jig.spmm_batched(b.hs[:n], b.dB[:n], b.dC[:n]), flush, pre=pre)
        print(json.dumps({"case": f"grouped c2 first {n} after a big-smem kernel", "event_us": us,
                          "cta_span_us": span(), "launch": jig.last_launch()}))
    us = timed(lambda: x.add_(1), flush, pre=pre)
    print(json.dumps({"case": "torch add_ after a big-smem kernel", "event_us": us}))


if __name__ == "__main__":
    main()
