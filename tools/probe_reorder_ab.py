"""Reorder device time and format hash per config (developer A/B of two builds via
JIGSAW_LIB_AB): the C2 points at s = .5/.7/.8 and the C2 batch total."""
import hashlib
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

tag = sys.argv[1] if len(sys.argv) > 1 else ""
torch.cuda.set_device(0)
tot, hs = 0.0, hashlib.blake2b(digest_size=8)
for i, (M, K, v, s, N) in enumerate(synth.c2_points()):
    A = synth.vector_sparse(M, K, v, s, 100 + i)
    a = torch.from_numpy(A.view(np.int16)).cuda().view(torch.float16)
    ms = []
    for rep in range(3):  # device times vary run to run; the minimum of three builds
        h = jig.reorder(a, v)
        ms.append(h.info()["reorder_ms"])
        if rep < 2:
            h.free()
    inf = dict(h.info(), reorder_ms=min(ms))
    g = h.export()
    d = hashlib.blake2b(digest_size=8)
    for k in ("T", "col_idx", "perm", "gather", "vals", "meta"):
        d.update(np.ascontiguousarray(g[k]).tobytes())
    hs.update(d.digest())
    tot += inf["reorder_ms"]
    if s <= 0.8:
        print(json.dumps({"tag": tag, "M": M, "K": K, "v": v, "s": s, "reorder_ms": inf["reorder_ms"],
                          "tiles": inf["ntiles"], "hash": d.hexdigest()}), flush=True)
    h.free()
print(json.dumps({"tag": tag, "c2_total_reorder_ms": tot, "hash": hs.hexdigest()}), flush=True)
