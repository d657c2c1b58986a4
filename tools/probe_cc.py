"""f3 measurement (DESIGN.md R-Q28): the C2 batch and its
single products with CUDA-core tiles at thresholds Z (cc_max_nnz), same box, L2
flushed before every step.  One JSON line per (scope, Z) on stdout.

  python tools/probe_cc.py [--z 0,16,32,64,128] [--workload c2]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--z", default="0,8,16,32,64,128")
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--singles", default="0.5,0.7", help="sparsities whose single products are timed")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream()
    flush = torch.empty(bench.FLUSH_BYTES, dtype=torch.uint8, device=dev)
    singles = [float(x) for x in a.singles.split(",") if x]
    for rep in range(2):
        for Z in [int(x) for x in a.z.split(",")]:
            b = bench.Batch(a.workload, 0, 1, 0, dev, torch, jig, cc_max_nnz=Z)
            ms, clk = bench.timed_steps(lambda: b.step(jig), a.steps, 5, flush, stream, torch)
            infos = [h.info() for h in b.hs]
            line = {"scope": "batch", "workload": a.workload, "rep": rep, "Z": Z, "us_per_step": ms * 1e3,
                    "tiles": sum(i["ntiles"] for i in infos), "cc_tiles": sum(i["cc_tiles"] for i in infos),
                    "cc_entries": sum(i["cc_entries"] for i in infos), "sm_mhz": clk.get("sm_mhz")}
            print(json.dumps(line), flush=True)
            if rep == 0:
                for h, dB, dC, (M, K, v, s, N) in zip(b.hs, b.dB, b.dC, b.points):
                    if s not in singles:
                        continue
                    us = bench.per_call_us(lambda h=h, dB=dB, dC=dC: h.spmm(dB, dC), flush, stream, torch)
                    inf = h.info()
                    print(json.dumps({"scope": "single", "Z": Z, "M": M, "K": K, "v": v, "s": s, "N": N,
                                      "us": us, "tiles": inf["ntiles"], "cc_tiles": inf["cc_tiles"],
                                      "cc_entries": inf["cc_entries"]}), flush=True)
            b.free()
            del b
            torch.cuda.synchronize()


if __name__ == "__main__":
    main()
