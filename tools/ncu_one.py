"""Launches one workload batch three times (L2 flushed before each) for an ncu
capture of the third k_spmm launch: ncu ... -k regex:k_spmm -s 2 -c 1 python
tools/ncu_one.py c2.  Developer tool."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
b = bench.Batch(sys.argv[1], 0, 1, int(sys.argv[2]) if len(sys.argv) > 2 else 0, dev, torch, jig)
for _ in range(3):
    flush.zero_()
    b.step(jig)
torch.cuda.synchronize()
print(jig.last_launch())
