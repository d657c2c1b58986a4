"""GPU probe (developer tool): one workload batch at one panel height / tile
width, timed like bench.py (events around a graph replay after an L2 flush) and
as a graph difference.  Usage: probe_c2_cfg.py <workload> <P> [tile_n] [tag]"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

name, P = sys.argv[1], int(sys.argv[2])
nt = int(sys.argv[3]) if len(sys.argv) > 3 else 0
tag = sys.argv[4] if len(sys.argv) > 4 else ""
torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
stream = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
b = bench.Batch(name, 0, 1, P, dev, torch, jig)
jig.set_launch_override(tile_n=nt, k_pieces=int(os.environ.get("KPIECES", "0")))
b.step(jig)
torch.cuda.synchronize()
d = jig.last_launch()
ms, clk = bench.timed_steps(lambda: b.step(jig), 30, 5, flush, stream, torch)
us = bench.per_call_us(lambda: b.step(jig), flush, stream, torch)
print(json.dumps({"tag": tag, "workload": name, "P": P, "nt": nt, "step_us": ms * 1e3, "graph_diff_us": us,
                  "pieces": d["split_slots"], "items": d["work_items"], "dyn": d["dynamic_schedule"],
                  "tile_n": d["tile_n"], "env": {k: v for k, v in os.environ.items() if k.startswith("JIGSAW_")}}))
