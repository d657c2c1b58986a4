"""Per-call wall times of jigsaw_spmm_batched_host on a bench batch (packed
pinned blocks, as bench.py), to separate per-call costs from box noise.
Developer tool: python tools/probe_e2e_calls.py c4 [calls]."""
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
dev = torch.device("cuda", 0)
w = sys.argv[1] if len(sys.argv) > 1 else "c4"
calls = int(sys.argv[2]) if len(sys.argv) > 2 else 15
b = bench.Batch(w, 0, 1, 0, dev, torch, jig)
nb = sum(B.size for (_, B) in b.mats)
nc = sum(M * N for (M, K, v, s, N) in b.points)
blk_b = torch.empty(nb, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
blk_c = torch.empty(nc, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
pB, pC, ob, oc = [], [], 0, 0
for (_, B), (M, K, v, s, N) in zip(b.mats, b.points):
    pB.append(blk_b[ob:ob + B.size].reshape(B.shape)); pB[-1][...] = B
    pC.append(blk_c[oc:oc + M * N].reshape(M, N)); ob += B.size; oc += M * N
ts = []
for _ in range(calls):
    t0 = time.perf_counter()
    jig.spmm_batched_host(b.hs, pB, pC)
    ts.append(round((time.perf_counter() - t0) * 1e3, 2))
# raw copy rates of the same blocks, for context
dB = torch.empty(nb, dtype=torch.int16, device=dev)
dC = torch.empty(nc, dtype=torch.int16, device=dev)
tb = torch.from_numpy(blk_b.view(np.int16)); tc = torch.from_numpy(blk_c.view(np.int16))
cp = []
for _ in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter(); dB.copy_(tb, non_blocking=True); torch.cuda.synchronize()
    t1 = time.perf_counter(); tc.copy_(dC, non_blocking=True); torch.cuda.synchronize(); t2 = time.perf_counter()
    cp.append((round(nb * 2 / (t1 - t0) / 1e9, 1), round(nc * 2 / (t2 - t1) / 1e9, 1)))
print(json.dumps({"workload": w, "lib": os.environ.get("JIGSAW_LIB_AB", "libjigsaw.so"), "call_ms": ts,
                  "h2d_d2h_GBps": cp}))
