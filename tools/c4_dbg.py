"""Grouped C4 launch time under the developer timing switches (JIGSAW_DBG, results
invalid): which data stream bounds the mainloop.  Developer tool."""
import os
import subprocess
import sys

code = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
import synth, paper_conf_icpp_zhanglyfyllq24_b200 as jig
from tools.time_c2 import med
torch.cuda.set_device(0)
wl = sys.argv[1]
pts = synth.c2_points() if wl == "c2" else synth.c4_points() if wl == "c4" else [(11008, 4096, 8, 0.9, 2048)]
dev = lambda x: torch.from_numpy(np.ascontiguousarray(x).view(np.int16)).cuda().view(torch.float16)
hs, Bs, Cs = [], [], []
for i, (M, K, v, s, N) in enumerate(pts):
    hs.append(jig.reorder(dev(synth.vector_sparse(M, K, v, s, 50 + i)), v, panel_rows=0))
    Bs.append(dev(synth.dense_b(K, N, 50 + i)))
    Cs.append(torch.empty((M, N), dtype=torch.float16, device="cuda"))
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
f = lambda: jig.spmm_batched(hs, Bs, Cs)
f(); torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    f()
torch.cuda.synchronize()
print(f"{wl} dbg={os.environ.get('JIGSAW_DBG','0')}: eager {med(f, flush)[0]:.1f} us, graph {med(g.replay, flush)[0]:.1f} us", flush=True)
'''
for wl in sys.argv[1:] or ["c4"]:
    for d in (os.environ.get("DBGS") or "0,2,8,16,24,26").split(","):
        env = dict(os.environ, JIGSAW_DBG=d)
        subprocess.run([sys.executable, "-c", code, wl], env=env)
