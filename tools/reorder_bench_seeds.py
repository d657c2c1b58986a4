"""Total GPU reorder device time of the bench's own C2 / C4 matrices (bench seeds).
Developer tool."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

torch.cuda.set_device(0)
for wl in ("c2", "c4"):
    pts = bench.workload(wl)[0] if isinstance(bench.workload(wl), tuple) else bench.workload(wl)
    tot, worst = 0.0, (0, None)
    for ji, p in enumerate(pts):
        M, K, v, s, N = p[:5]
        seed = bench.point_seed(ji, 0)
        A = bench.make_a(wl, ji, M, K, v, s, seed)
        h = jig.reorder(torch.from_numpy(A.view(np.int16)).cuda().view(torch.float16), v, panel_rows=0)
        ms = h.info()["reorder_ms"]
        tot += ms
        worst = max(worst, (ms, (M, K, v, s)))
        h.free()
    print(f"{wl}: reorder total {tot:.0f} ms, worst {worst[0]:.0f} ms at {worst[1]}", flush=True)
