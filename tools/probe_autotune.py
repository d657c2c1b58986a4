"""Which panel height the autotune (panel_rows = -1) keeps for the C2 and C4
points (probe product N = the workload's N).  Developer tool; prints JSON lines."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

torch.cuda.set_device(0)
for w in ("c2", "c4"):
    pts, _, _ = bench.workload(w)
    for i, (M, K, v, s, N) in enumerate(pts):
        A = bench.make_a(w, i, M, K, v, s, bench.point_seed(i, 0))
        a = torch.from_numpy(A.view(np.int16)).cuda().view(torch.float16)
        h = jig.reorder(a, v, panel_rows=jig.PANEL_AUTOTUNE, autotune_n=N)
        inf = h.info()
        print(json.dumps({"workload": w, "M": M, "K": K, "v": v, "s": s, "N": N, "chosen_P": inf["panel_rows"],
                          "reorder_ms_incl_autotune": round(inf["reorder_ms"], 2)}))
        h.free()
