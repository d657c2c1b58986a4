"""GPU probe (developer tool): the C2 batch step at panel heights 128 / 256 and
tile widths / piece splitting, timed like bench.py (events around a graph
replay, L2 flushed before).  Prints one JSON object."""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
stream = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
which = sys.argv[1] if len(sys.argv) > 1 else "c2"
out = {}
for P in (128, 256):
    b = bench.Batch(which, 0, 1, P, dev, torch, jig)
    out[f"P{P}_ntiles"] = sum(h.info()["ntiles"] for h in b.hs)
    for nt in (0, 128, 256):
        for nop in (0, 1):
            if P == 128 and nt == 256:
                continue
            with jig.launch_override(tile_n=nt, no_pieces=nop):
                b.step(jig)
                torch.cuda.synchronize()
                d = jig.last_launch()
                ms, clk = bench.timed_steps(lambda: b.step(jig), 30, 5, flush, stream, torch)
                us = bench.per_call_us(lambda: b.step(jig), flush, stream, torch)
            out[f"P{P}_nt{nt}_nopieces{nop}"] = {"step_ms": ms, "graph_diff_us": us, "tile_n": d["tile_n"],
                                                 "pieces": d["split_slots"], "items": d["work_items"],
                                                 "dyn": d["dynamic_schedule"], "grid": d["grid"]}
            print(P, nt, nop, out[f"P{P}_nt{nt}_nopieces{nop}"], file=sys.stderr)
    b.free()
print(json.dumps(out))
