"""GPU probe (developer tool): C2 batch -- jigsaw grouped step (dynamic vs static
schedule) against batched and per-matrix cuBLAS (16F / 32F compute), L2 flushed.
Prints one JSON object."""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from tools import cublas_ref  # noqa: E402

torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
stream = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
pts = synth.c2_points()
dA, dB, dC, hs = [], [], [], []
for i, (M, K, v, s, N) in enumerate(pts):
    A = synth.vector_sparse(M, K, v, s, synth.SEED_BASE + i)
    B = synth.dense_b(K, N, synth.SEED_BASE + i)
    a = torch.from_numpy(A.view(np.int16)).to(dev).view(torch.float16)
    dA.append(a)
    dB.append(torch.from_numpy(B.view(np.int16)).to(dev).view(torch.float16))
    dC.append(torch.empty((M, N), dtype=torch.float16, device=dev))
    hs.append(jig.reorder(a, v))
R, REPS = 8, 9


def graphed(fn):
    if fn is not None:
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(R):
            flush.zero_()
            if fn is not None:
                fn()
    return g


def timeit(g):
    ts = []
    for _ in range(REPS):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        g.replay()
        e1.record(stream)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


t0 = timeit(graphed(None))


def per_call_us(fn):
    return (timeit(graphed(fn)) - t0) / R * 1e3


out = {}
out["jigsaw_step_us"] = per_call_us(lambda: jig.spmm_batched(hs, dB, dC))
os.environ["JIGSAW_STATIC_SCHEDULE"] = "1"
out["jigsaw_step_static_rr_us"] = per_call_us(lambda: jig.spmm_batched(hs, dB, dC))
del os.environ["JIGSAW_STATIC_SCHEDULE"]
# batched cuBLAS per shape group
groups = {}
for i, (M, K, v, s, N) in enumerate(pts):
    groups.setdefault((M, K, N), []).append(i)
stk = {}
for key, idx in groups.items():
    M, K, N = key
    stk[key] = (torch.stack([dA[i] for i in idx]), torch.stack([dB[i] for i in idx]),
                torch.empty((len(idx), M, N), dtype=torch.float16, device=dev))
for comp in ("16F", "32F"):
    def step(comp=comp):
        for A3, B3, C3 in stk.values():
            cublas_ref.gemm_strided_batched(A3, B3, C3, comp)
    out[f"cublas_strided_batched_{comp}_us"] = per_call_us(step)


def bmm_step():
    for A3, B3, C3 in stk.values():
        torch.bmm(A3, B3, out=C3)


out["torch_bmm_us"] = per_call_us(bmm_step)
Cs = [torch.empty_like(c) for c in dC]


def serial(comp):
    def f():
        for a, b, c in zip(dA, dB, Cs):
            cublas_ref.gemm(a, b, c, comp)
    return f


out["cublas_serial_16F_us"] = per_call_us(serial("16F"))
out["cublas_serial_32F_us"] = per_call_us(serial("32F"))
per = []
for i, (M, K, v, s, N) in enumerate(pts):
    d = {"tag": f"{M}x{K}_v{v}_s{int(s*100)}"}
    d["jig"] = per_call_us(lambda: hs[i].spmm(dB[i], C=dC[i]))
    d["c16"] = per_call_us(lambda: cublas_ref.gemm(dA[i], dB[i], Cs[i], "16F"))
    d["c32"] = per_call_us(lambda: cublas_ref.gemm(dA[i], dB[i], Cs[i], "32F"))
    d["mm"] = per_call_us(lambda: torch.matmul(dA[i], dB[i], out=Cs[i]))
    per.append(d)
out["per_matrix"] = per
out["info"] = [{k: h.info()[k] for k in ("M","K","ntiles","kp_total","nksteps","evictions","overflow_tiles","max_tiles")} for h in hs]
# correctness spot-check of the baseline binding
ref = torch.matmul(dA[3].float(), dB[3].float())
cublas_ref.gemm(dA[3], dB[3], Cs[3], "32F")
out["cublas_binding_maxerr"] = float((Cs[3].float() - ref).abs().max())
print(json.dumps(out))
