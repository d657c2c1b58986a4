"""Step time with the L2 flushed before every step (the bench's rule) vs warm (no
flush: the previous step's A, B and C partly in L2).  Developer tool: how much of
the k-block time is DRAM first-touch latency."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
stream = torch.cuda.current_stream()
flush = torch.empty(bench.FLUSH_BYTES, dtype=torch.uint8, device=dev)
tiny = torch.empty(1024, dtype=torch.uint8, device=dev)   # a "flush" that flushes nothing
for name in sys.argv[1:] or ["c2", "c4"]:
    b = bench.Batch(name, 0, 1, 0, dev, torch, jig)
    for rep in range(2):
        cold, _ = bench.timed_steps(lambda: b.step(jig), 20, 5, flush, stream, torch)
        warm, _ = bench.timed_steps(lambda: b.step(jig), 20, 5, tiny, stream, torch)
        print(json.dumps({"workload": name, "cold_us": cold * 1e3, "warm_us": warm * 1e3,
                          "alg_MB": b.alg_bytes / 1e6}), flush=True)
    b.free()
