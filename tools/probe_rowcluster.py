"""GPU study (developer tool): row-clustered panels vs the given
row order on C2-shaped batches with uniform and skewed (magnitude-pruned-like)
row densities: tiles, K_p, reorder time, and the grouped-step time (graph
difference, L2 flushed).  Prints JSON lines."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
stream = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
for kind in ("uniform", "skewed"):
    pts = synth.c2_points()
    As = [synth.vector_sparse(M, K, v, s, synth.SEED_BASE + i, kind=kind) for i, (M, K, v, s, N) in enumerate(pts)]
    dB = [torch.from_numpy(synth.dense_b(K, N, synth.SEED_BASE + i).view(np.int16)).to(dev).view(torch.float16)
          for i, (M, K, v, s, N) in enumerate(pts)]
    dC = [torch.empty((M, N), dtype=torch.float16, device=dev) for (M, K, v, s, N) in pts]
    for ro in (0, 1):
        hs = [jig.reorder(torch.from_numpy(A.view(np.int16)).to(dev).view(torch.float16), v, row_order=ro)
              for A, (M, K, v, s, N) in zip(As, pts)]
        inf = [h.info() for h in hs]
        us = bench.per_call_us(lambda: jig.spmm_batched(hs, dB, dC), flush, stream, torch)
        per = {}
        for h, (M, K, v, s, N), i in zip(hs, pts, inf):
            per.setdefault(f"v{v}_s{int(s*100)}", []).append(i["ntiles"])
        print(json.dumps({"kind": kind, "row_order": ro, "step_us": us,
                          "ntiles": sum(i["ntiles"] for i in inf), "kp_total": sum(i["kp_total"] for i in inf),
                          "reorder_ms": sum(i["reorder_ms"] for i in inf), "tiles_by_v_s": per}))
        for h in hs:
            h.free()
