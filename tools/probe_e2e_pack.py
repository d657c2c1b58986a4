"""e2e host-buffer batch (jigsaw_spmm_batched_host): separate pinned buffers per
product vs the batch packed in one pinned block per direction.  Developer tool."""
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
for w in sys.argv[1:] or ["c2", "c4"]:
    b = bench.Batch(w, 0, 1, 0, dev, torch, jig)
    sep_B = [torch.from_numpy(B.view(np.int16)).pin_memory().numpy().view(np.uint16) for (_, B) in b.mats]
    sep_C = [torch.empty((M, N), dtype=torch.int16).pin_memory().numpy().view(np.uint16) for (M, K, v, s, N) in b.points]
    nb = sum(B.size for (_, B) in b.mats)
    nc = sum(M * N for (M, K, v, s, N) in b.points)
    blk_b = torch.empty(nb, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
    blk_c = torch.empty(nc, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
    pk_B, pk_C, ob, oc = [], [], 0, 0
    for (_, B), (M, K, v, s, N) in zip(b.mats, b.points):
        pk_B.append(blk_b[ob:ob + B.size].reshape(B.shape)); pk_B[-1][...] = B
        pk_C.append(blk_c[oc:oc + M * N].reshape(M, N)); ob += B.size; oc += M * N
    res = {}
    variants = (("separate", (sep_B, sep_C)), ("packed", (pk_B, pk_C)),
                ("packed_B_only", (pk_B, sep_C)), ("packed_C_only", (sep_B, pk_C)))
    for rep in range(int(os.environ.get("REPS", "3"))):
        for name, (Bs, Cs) in variants:
            jig.spmm_batched_host(b.hs, Bs, Cs)
            t0 = time.perf_counter()
            for _ in range(5):
                jig.spmm_batched_host(b.hs, Bs, Cs)
            res.setdefault(name, []).append((time.perf_counter() - t0) / 5 * 1e3)
    print(json.dumps({"workload": w, "ms_per_step": {k: [round(x, 3) for x in v] for k, v in res.items()}}))
    b.free()
