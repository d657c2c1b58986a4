"""One GPU reorder (for ncu launch lists of R1-R5).  Developer tool."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools.trace_spmm import dev  # noqa: E402

M, K, v, s = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), float(sys.argv[4])
h = jig.reorder(dev(synth.vector_sparse(M, K, v, s, 91)), v, panel_rows=0)
torch.cuda.synchronize()
print(h.info()["reorder_ms"])
