"""Reorder throughput of a batch (developer tool): the 36 C2 matrices built one
jigsaw_reorder_ex at a time vs one jigsaw_reorder_batched call (wall clock)."""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

torch.cuda.set_device(0)
for w in ("c2", "c4"):
    pts, _, _ = bench.workload(w)
    dA = [torch.from_numpy(bench.make_a(w, i, M, K, v, s, bench.point_seed(i, 0)).view(np.int16)).cuda()
          .view(torch.float16) for i, (M, K, v, s, N) in enumerate(pts)]
    vs = [v for (M, K, v, s, N) in pts]
    for rep in range(2):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        hs = [jig.reorder(a, v, panel_rows=0) for a, v in zip(dA, vs)]
        t1 = time.perf_counter()
        dev_ms = sum(h.info()["reorder_ms"] for h in hs)
        for h in hs:
            h.free()
        t2 = time.perf_counter()
        hb = jig.reorder_batched(dA, vs, panel_rows=0)
        t3 = time.perf_counter()
        for h in hb:
            h.free()
    print(json.dumps({"workload": w, "matrices": len(pts), "sequential_wall_ms": (t1 - t0) * 1e3,
                      "sequential_device_ms_sum": dev_ms, "batched_wall_ms": (t3 - t2) * 1e3}))
