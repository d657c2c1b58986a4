"""GPU probe (developer tool): isolated C2 products (graph difference, L2 flushed
before every call): jigsaw at the library's choice and at forced tile / split
variants, vs cuBLAS (best of 16F / 32F).  Prints JSON lines."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools import cublas_ref  # noqa: E402

torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
stream = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
variants = [dict()] + ([dict(tile_n=nt, split_k=s) for nt in (32, 64) for s in (1, 2, 4, 8)]
                       if "--variants" in sys.argv else [])
for (M, K, v, s) in [(512, 2048, 4, 0.9), (512, 2048, 8, 0.9), (2048, 512, 4, 0.9), (2048, 512, 8, 0.95),
                     (512, 2048, 8, 0.98), (2048, 512, 2, 0.5)]:
    N = 256
    A = synth.vector_sparse(M, K, v, s, 5)
    dA = torch.from_numpy(A.view(np.int16)).to(dev).view(torch.float16)
    dB = torch.from_numpy(synth.dense_b(K, N, 5).view(np.int16)).to(dev).view(torch.float16)
    C = torch.empty((M, N), dtype=torch.float16, device=dev)
    h = jig.reorder(dA, v)
    row = {"shape": f"{M}x{K}_v{v}_s{int(s*100)}",
           "cublas": min(bench.per_call_us(lambda: cublas_ref.gemm(dA, dB, C, c), flush, stream, torch)
                         for c in ("16F", "32F"))}
    for ov in variants:
        with jig.launch_override(**ov):
            h.spmm(dB, C=C)
            d = jig.last_launch()
            t = bench.per_call_us(lambda: h.spmm(dB, C=C), flush, stream, torch)
        row["jig" + "".join(f"_{k}{v_}" for k, v_ in ov.items())] = round(t, 2)
        if not ov:
            row["choice"] = f"NT{d['tile_n']} S{d['split_k']} grid{d['grid']}"
    print(json.dumps(row))
