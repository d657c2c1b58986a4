#!/usr/bin/env python
"""bench.py -- SpMM effective TFLOP/s and speedup vs cuBLAS fp16 GEMM vs sparsity
(BASELINE.json metric) for the Jigsaw hot path on B200.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c2|c1|c3|c4|c5a|c5b|venom]
                  [--impl jigsaw|reference]

A STEP is one pass of the SpMM hot path over one batch of synthetic matrices
with the prepared formats resident in HBM (the paper times the kernel only and
excludes format conversion): for the default workload (BASELINE
configs[1], "C2") the batch is the 36 DLMC-transformer-shaped matrices
512x2048 / 2048x512 x v in {2,4,8} x s in {.50,.70,.80,.90,.95,.98}, N = 256.
  value   = sum over the batch of 2*M*N*K (dense-equivalent flops) / step time
  e2e     = the same metric through the C ABI with HOST buffers
            (jigsaw_spmm_batched_host: the batch's B's host->device, grouped SpMM,
            C's device->host, every step; chunks overlap on three streams)
  e2e_full= + the reorder of A from host memory (jigsaw_reorder_host) every step,
            i.e. every §8(a) row of the hot path
L2 is flushed (256 MB write) before every timed step; per-step device time is
taken with CUDA events on the launching stream and summed; multi-GPU: one
process per GPU (torchrun), weak scaling (each rank its own batch, seeds offset
by rank), barrier + synchronize around the timed region, max over ranks.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "SpMM effective TFLOP/s and speedup vs cuBLAS fp16 GEMM vs sparsity, v=2/4/8"
FLUSH_BYTES = 256 << 20


# ------------------------------------------------------------------ workloads
def workload(name: str):
    """(points, description, scaling).  A point is (M, K, v, s, N)."""
    if name == "c2":
        return synth.c2_points(), ("C2: DLMC-transformer A 512x2048 and 2048x512, v=2/4/8, "
                                   "s=.50/.70/.80/.90/.95/.98, N=256 (36 matrices)"), "weak"
    if name == "c1":
        c = synth.C1
        return [(c["M"], c["K"], c["v"], c["s"], c["N"])], "C1: 256x256 v=4 s=.80 N=64", "weak"
    if name == "c3":
        pts = [(M, K, v, s, N) for (M, K) in synth.C3_SHAPES for v in synth.C3_V for s in synth.C3_S
               for N in synth.C3_N]
        return pts, ("C3: ResNet-50 conv-as-GEMM layers (19 shapes) x v=4/8 x s=.70/.80/.90/.95 x "
                     "N=256/1024 (304 matrices)"), "weak"
    if name == "c4":
        return synth.c4_points(), ("C4: pruned Llama linear 4096x4096 and 11008x4096, v=8, "
                                   "s=.50/.70/.80/.90, N=2048 (8 matrices)"), "weak"
    if name == "c5a":
        L = synth.C2_SHAPES + synth.C3_SHAPES
        pts = [(L[i % len(L)][0], L[i % len(L)][1], (4, 8)[i % 2], (0.7, 0.8, 0.9, 0.95)[(i // 2) % 4], 256)
               for i in range(64)]
        return pts, ("C5a: batch of 64 DLMC-shaped matrices (C2 + C3 shapes), v=4/8, s=.7-.95, N=256, "
                     "sharded by matrix (LPT) across the GPUs"), "strong"
    if name == "c5b":
        return [(4096, 4096, 8, 0.90, 16384)], ("C5b: 4096x4096 v=8 s=.90 N=16384, B/C column-sharded "
                                                "across the GPUs"), "strong"
    if name == "venom":
        # SURVEY §8f f4 (Table 3): matrices already pruned to V:2:Mb,
        # computed without a reorder step being needed; v = 1 (the format is
        # v-independent), s = 1 - 2/Mb
        pts = [(M, K, 1, 1.0 - 2.0 / mb, N) for (M, K, V, mb, N) in synth.venom_points()]
        return pts, ("f4: VENOM-style V:2:Mb pruned 4096x4096, V=32/64/128, Mb=12/20/40/100 "
                     "(s=.833/.90/.95/.98), N=2048 (12 matrices), vs cuBLAS and cuSPARSELt"), "weak"
    raise SystemExit(f"unknown workload {name}")


def make_a(name: str, i: int, M: int, K: int, v: int, s: float, seed: int) -> np.ndarray:
    """A of point i of workload `name` (uint16 fp16 bits)."""
    if name == "venom":
        _, _, V, mb, _ = synth.venom_points()[i]
        return synth.venom(M, K, V, mb, seed)
    return synth.vector_sparse(M, K, v, s, seed)


def point_tag(name: str, i: int, v: int, s: float) -> str:
    if name == "venom":
        _, _, V, mb, _ = synth.venom_points()[i]
        return f"V{V}_Mb{mb}"
    return f"v{v}_s{int(round(s * 100))}"


def local_jobs(name, points, rank, world):
    """This rank's share of the workload: list of (M, K, v, s, N, seed, n0, n1).
    Weak workloads: every point, seeds offset by rank.  c5a: matrices assigned by
    LPT on the dense-equivalent work.  c5b: the same A on every rank, columns
    [n0, n1) of one B (paper_conf_icpp_zhanglyfyllq24_b200.shard)."""
    from paper_conf_icpp_zhanglyfyllq24_b200 import shard
    if name == "c5a":
        costs = [2.0 * M * K * N * (1 - s) for (M, K, v, s, N) in points]
        mine = shard.lpt_assign(costs, world)[rank]
        return [(*points[i], point_seed(i, 0), 0, points[i][4]) for i in mine]
    if name == "c5b":
        (M, K, v, s, N), = points
        n0, n1 = shard.column_shards(N, world)[rank]
        return [(M, K, v, s, N, point_seed(0, 0), n0, n1)] if n1 > n0 else []
    return [(M, K, v, s, N, point_seed(i, rank), 0, N) for i, (M, K, v, s, N) in enumerate(points)]


def point_seed(i: int, rank: int) -> int:
    return synth.SEED_BASE + 1000 * rank + i


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), float(d["bf16_tflops"]), "measured"
    except Exception:
        return 6650.0, 1590.0, "fallback (B200_PROFILING.md)"


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks and throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index, self.rows, self.proc = index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 6:
                self.rows.append(parts)

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.12)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=1)
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[2 + i] == "Active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(self.rows)}


# ------------------------------------------------------------------ roofline terms
def algorithmic(info: dict, M: int, K: int, N: int, rows_touched: int):
    """Per-launch algorithmic bytes and executed flops of k_spmm."""
    P = info["panel_rows"]
    n_tiles = (N + 127) // 128
    a_bytes = (16 * P + 2 * P + 64) * info["ntiles"]          # values + metadata + gather per tile
    b_bytes = 2 * N * rows_touched                              # touched B rows, once
    c_bytes = 2 * M * N
    exec_flops = 2 * P * 16 * info["ntiles"] * N               # logical sparse MMA work
    return a_bytes + b_bytes + c_bytes, exec_flops, n_tiles


# ------------------------------------------------------------------ reference arm (CPU oracle)
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    points, desc, scaling = workload(args.workload)
    cores = 1
    try:
        os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})
    except Exception:
        cores = 1
    mats = [(make_a(args.workload, i, M, K, v, s, point_seed(i, 0)), synth.dense_b(K, N, point_seed(i, 0)))
            for i, (M, K, v, s, N) in enumerate(points)]
    # size the per-step sample so the whole run stays within ~2 minutes
    budget = max(0.2, min(4.0, 100.0 / max(1, args.steps + args.warmup)))
    t0 = time.perf_counter()
    oracle.spmm(mats[0][0], mats[0][1], rows=[0])
    per_row = (time.perf_counter() - t0)
    rows_per_point = max(1, int(budget / max(per_row * len(points), 1e-6)))
    rows_per_point = min(rows_per_point, min(M for (M, K, v, s, N) in points))

    def step():
        fl = 0
        for (A, B), (M, K, v, s, N) in zip(mats, points):
            oracle.spmm(A, B, rows=list(range(rows_per_point)))
            fl += 2 * rows_per_point * N * K
        return fl

    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    fl = sum(step() for _ in range(args.steps))
    dt = time.perf_counter() - t0
    val = fl / dt / 1e12
    sample = f"first {rows_per_point} rows of each of the {len(points)} matrices, full N"
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "TFLOP/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": dt / args.steps * 1e3, "higher_is_better": True, "scaling": scaling,
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": desc, "l2": "n/a (CPU)"},
            "cpu_baseline": {"value": val, "unit": "TFLOP/s", "cores": cores, "kind": "oracle",
                             "sample": sample, "cpu_model": cpu_model()},
            "e2e": {"value": val, "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


def cpu_baseline(points, mats, budget_s=12.0):
    """The oracle (plain C, fp64, single thread) on a bounded sample of the same workload."""
    import oracle
    try:
        os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})
    except Exception:
        pass
    t0 = time.perf_counter()
    oracle.spmm(mats[0][0], mats[0][1], rows=[0])
    per_row = time.perf_counter() - t0
    rows = max(1, int(budget_s / max(per_row * len(points), 1e-6)))
    rows = min(rows, min(M for (M, K, v, s, N) in points))
    fl = 0
    t0 = time.perf_counter()
    for (A, B), (M, K, v, s, N) in zip(mats, points):
        oracle.spmm(A, B, rows=list(range(rows)))
        fl += 2 * rows * N * K
    dt = time.perf_counter() - t0
    return {"value": fl / dt / 1e12, "unit": "TFLOP/s", "cores": 1, "kind": "oracle",
            "sample": f"first {rows} rows of each of the {len(points)} matrices, full N "
                      f"({dt:.1f} s of CPU work)", "cpu_model": cpu_model()}


def cpu_model() -> str:
    """Host CPU model (the CPU baseline's hardware)."""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


# ------------------------------------------------------------------ jigsaw arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--panel-rows", type=int, default=0, choices=[0, 128, 256],
                    help="reorder panel height: 0 = library auto (256 for M >= 4096), 128 (one CTA "
                         "per panel) or 256 (CTA pairs)")
    ap.add_argument("--impl", default="jigsaw", choices=["jigsaw", "reference"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-cublas", action="store_true")
    ap.add_argument("--detail", action="store_true", help="print the per-point table to stderr")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    import paper_conf_icpp_zhanglyfyllq24_b200 as jig

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    stream = torch.cuda.current_stream()
    hbm, bf16, peak_src = load_peaks()

    all_points, desc, scaling = workload(args.workload)
    jobs = local_jobs(args.workload, all_points, rank, world)
    points = [(M, K, v, s, n1 - n0) for (M, K, v, s, N, seed, n0, n1) in jobs]
    total_eff = sum(2 * M * K * N for (M, K, v, s, N) in all_points) * (world if scaling == "weak" else 1)
    mats, hs, dB, dC, dA = [], [], [], [], []
    reorder_ms = 0.0
    alg_bytes = exec_flops = eff_flops = 0
    for ji, (M, K, v, s, N, seed, n0, n1) in enumerate(jobs):
        A = make_a(args.workload, ji, M, K, v, s, seed)
        B = synth.dense_b(K, N, seed)
        if (n0, n1) != (0, N):
            B = np.ascontiguousarray(B[:, n0:n1])
        N = n1 - n0
        mats.append((A, B))
        a_t = torch.from_numpy(A.view(np.int16)).to(dev).view(torch.float16)
        h = jig.reorder(a_t, v, panel_rows=args.panel_rows)
        info = h.info()
        reorder_ms += info["reorder_ms"]
        hs.append(h)
        dA.append(a_t)
        dB.append(torch.from_numpy(B.view(np.int16)).to(dev).view(torch.float16))
        dC.append(torch.empty((M, N), dtype=torch.float16, device=dev))
        rows_touched = int(((A & 0x7FFF) != 0).any(axis=0).sum())
        ab, ef, _ = algorithmic(info, M, K, N, rows_touched)
        alg_bytes += ab
        exec_flops += ef
        eff_flops += 2 * M * N * K
    flush = torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev)

    def step_eager():
        # the whole batch in grouped launches (jigsaw_spmm_batched: <= 64 products per kernel)
        jig.spmm_batched(hs, dB, dC)

    def step_unbatched():
        for h, b, c in zip(hs, dB, dC):
            h.spmm(b, C=c)

    # warm up eagerly (first-call attribute setup), then capture the step in a CUDA
    # graph so that host launch latency stays out of the device timing
    for _ in range(2):
        step_eager()
        step_unbatched()
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph):
        step_eager()
    graph_unb = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph_unb):
        step_unbatched()
    torch.cuda.synchronize()
    launches = (len(points) + 63) // 64

    def step():
        graph.replay()

    for _ in range(args.warmup):
        flush.zero_()
        step()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(args.steps)]
    sampler = ClockSampler(dev.index if dev.index is not None else 0)
    sampler.start()
    time.sleep(0.15)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for k in range(args.steps):
        flush.zero_()                     # L2 flush, outside the timed events
        evs[k][0].record(stream)
        step()
        evs[k][1].record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    total_ms = sum(a.elapsed_time(b) for a, b in evs)
    t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    value = total_eff / (ms_per_step * 1e-3) / 1e12   # whole job, all ranks

    # roofline of the dominant (only) kernel, k_spmm: algorithmic bytes / flops per
    # launch over the average launch duration of the timed region
    t_hbm = alg_bytes / (hbm * 1e9)
    t_tc = exec_flops / (2 * bf16 * 1e12)          # sparse logical peak = 2x dense
    if t_hbm >= t_tc:
        roof = {"bound": "hbm", "achieved": alg_bytes / (ms_per_step * 1e-3) / 1e9, "peak": hbm,
                "unit": "GB/s"}
    else:
        roof = {"bound": "tensor", "achieved": exec_flops / (ms_per_step * 1e-3) / 1e12,
                "peak": 2 * bf16, "unit": "TFLOP/s"}
    roof["frac"] = roof["achieved"] / roof["peak"]
    roof["peak_source"] = peak_src
    roof["traffic"] = None
    roof["per_launch_us"] = ms_per_step * 1e3 / launches
    roof["t_roof_us_per_step"] = max(t_hbm, t_tc) * 1e6
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))[args.workload]
        roof["traffic"] = prof["bytes_per_step"] / launches
        roof["traffic_unit"] = "bytes per launch"
        roof["traffic_source"] = prof.get("source")
    except Exception:
        pass

    # per-point detail: jigsaw vs cuBLAS (torch.matmul on the dense fp16 A).  Each
    # call's device time in a stream of back-to-back kernels, L2 flushed before
    # every call: [graph of R x (flush, call)] - [graph of R x (flush)], / R (median
    # of reps) -- the event clock here moves in ~2 us steps, too coarse for
    # single-call events; the difference over R calls resolves ~0.1 us.
    detail = []
    cublas_ms = jig_ms = cslt_ms = 0.0
    # cuSPARSELt (torch._cslt_*) on natively 2:4 inputs (the f4 workload): the
    # library 2:4 SpMM, which cannot skip all-zero columns
    cslt_A, cslt_err = None, None
    if not args.no_cublas and args.workload == "venom":
        try:
            cslt_A = [torch._cslt_compress(a) for a in dA]
            torch._cslt_sparse_mm(cslt_A[0], dB[0])
            torch.cuda.synchronize()
        except Exception as e:  # library without an sm_100 build, or API absent
            cslt_A, cslt_err = None, f"{type(e).__name__}: {str(e).splitlines()[0][:200]}"
    if not args.no_cublas:
        reps, R = 7, 8

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
            for _ in range(reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                g.replay()
                e1.record(stream)
                e1.synchronize()
                ts.append(e0.elapsed_time(e1))
            return float(np.median(ts))
        g_flush = graphed(None)
        for i, (M, K, v, s, N) in enumerate(points):
            t0 = timeit(g_flush)
            tj = (timeit(graphed(lambda: hs[i].spmm(dB[i], C=dC[i]))) - t0) / R
            Cref = torch.empty_like(dC[i])
            tc = (timeit(graphed(lambda: torch.matmul(dA[i], dB[i], out=Cref))) - t0) / R
            cublas_ms += tc
            jig_ms += tj
            d = {"M": M, "K": K, "v": v, "s": s, "N": N, "tag": point_tag(args.workload, i, v, s),
                 "jigsaw_us": tj * 1e3, "cublas_us": tc * 1e3, "speedup": tc / tj,
                 "eff_tflops": 2 * M * N * K / (tj * 1e-3) / 1e12}
            if cslt_A is not None and cslt_A[i] is not None:
                ts = (timeit(graphed(lambda: torch._cslt_sparse_mm(cslt_A[i], dB[i]))) - t0) / R
                d["cusparselt_us"] = ts * 1e3
                d["speedup_vs_cusparselt"] = ts / tj
                cslt_ms += ts
            detail.append(d)
    # step-level comparison: the same batch as one CUDA graph of per-matrix cuBLAS
    # calls, and of per-matrix jigsaw_spmm calls (36 launches), same flush policy
    def step_ms(g, reps=30):
        ts = []
        for _ in range(reps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            g.replay()
            e1.record(stream)
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        return float(np.median(ts))
    outs = [torch.empty_like(c) for c in dC]

    def cublas_step():
        for a, b, o in zip(dA, dB, outs):
            torch.matmul(a, b, out=o)
    cublas_step()
    torch.cuda.synchronize()
    g_cub = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g_cub):
        cublas_step()
    cublas_step_ms = step_ms(g_cub)
    unbatched_step_ms = step_ms(graph_unb)
    speed = {}
    speed_cs = {}
    for d in detail:
        speed.setdefault(d["tag"], []).append(d["speedup"])
        if "speedup_vs_cusparselt" in d:
            speed_cs.setdefault(d["tag"], []).append(d["speedup_vs_cusparselt"])
    speed_gm = {k: float(np.exp(np.mean(np.log(x)))) for k, x in sorted(speed.items())}
    cslt = None
    if cslt_A is not None:
        def cslt_step():
            for a, b, o in zip(cslt_A, dB, outs):
                o.copy_(torch._cslt_sparse_mm(a, b))
        cslt_step()
        torch.cuda.synchronize()
        g_cs = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g_cs):
            cslt_step()
        cs_ms = step_ms(g_cs)
        cslt = {"step_ms": cs_ms, "speedup_step": cs_ms / ms_per_step,
                "speedup_total_time": (cslt_ms / jig_ms) if jig_ms else None,
                "speedup_geomean_by_point": {k: float(np.exp(np.mean(np.log(x)))) for k, x in sorted(speed_cs.items())},
                "how": "torch._cslt_compress / torch._cslt_sparse_mm (cuSPARSELt 2:4 SpMM) on the natively 2:4 A; "
                       "per matrix like cuBLAS; step = one CUDA graph of the batch (+ a copy into C per matrix)"}
    elif cslt_err:
        cslt = {"unavailable": cslt_err}

    # e2e through the C ABI with host buffers (every step: B in, SpMM, C out)
    pin_B = [torch.from_numpy(B.view(np.int16)).pin_memory().numpy().view(np.uint16) for (_, B) in mats]
    pin_C = [torch.empty((M, N), dtype=torch.int16).pin_memory().numpy().view(np.uint16)
             for (M, K, v, s, N) in points]
    h2d = sum(B.nbytes for (_, B) in mats)
    d2h = sum(2 * M * N for (M, K, v, s, N) in points)
    e2e_steps = max(3, min(args.steps, 20))
    # one jigsaw_spmm_batched_host call per step: copy-in, grouped SpMM and
    # copy-out of successive chunks of the batch overlap on three streams
    jig.spmm_batched_host(hs, pin_B, pin_C)
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(e2e_steps):
        jig.spmm_batched_host(hs, pin_B, pin_C)
    e2e_s = (time.perf_counter() - t0) / e2e_steps
    te = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_s = float(te.item())
    # e2e_full: host A -> reorder -> host B -> SpMM -> host C (all §8(a) rows)
    t0 = time.perf_counter()
    for (A, B), (M, K, v, s, N) in zip(mats, points):
        hh = jig.reorder_host(A, v, panel_rows=args.panel_rows)
        hh.spmm_host(B)
        hh.free()
    full_s = time.perf_counter() - t0

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline(points, mats)

    line = {
        "metric": METRIC, "value": value, "unit": "TFLOP/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
        "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "f16",
        "data": "synthetic",
        "config": {"workload": desc, "matrices_on_rank0": len(points),
                   "flops": "dense-equivalent 2*M*N*K per matrix",
                   "l2": "flushed (256 MB write) before every timed step", "launch": "step = jigsaw_spmm_batched over the batch (one grouped k_spmm launch per 64 matrices), captured in a CUDA graph",
                   "seeds": f"synth.SEED_BASE + 1000*rank + index", "format": f"panel_rows={args.panel_rows or 'auto'} (P used: {sorted(set(h.info()['panel_rows'] for h in hs))}), SPTC residual"},
        "roofline": roof,
        "cpu_baseline": cpu,
        "e2e": {"value": total_eff / e2e_s / 1e12, "unit": "TFLOP/s",
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "call": "jigsaw_spmm_batched_host (pinned host buffers), wall clock per step"},
        "e2e_full": {"value": eff_flops / full_s / 1e12, "unit": "TFLOP/s",
                     "note": "rank 0: jigsaw_reorder_host + jigsaw_spmm_host per matrix, one pass"},
        "gpu_launches": launches * args.steps,
        "clocks": clocks,
        "cublas": {"step_ms": cublas_step_ms, "step_tflops": eff_flops / (cublas_step_ms * 1e-3) / 1e12,
                   "speedup_step": cublas_step_ms / ms_per_step,
                   "jigsaw_unbatched_step_ms": unbatched_step_ms,
                   "speedup_total_time": (cublas_ms / jig_ms) if jig_ms else None,
                   "speedup_geomean_by_v_s": speed_gm,
                   "cublas_eff_tflops": (eff_flops / (cublas_ms * 1e-3) / 1e12) if cublas_ms else None,
                   "how": "torch.matmul fp16 (cuBLAS) on the dense A: per matrix as [graph of 8 x (L2 flush, call)] - [graph of 8 x (L2 flush)], / 8 (median of 7), and the whole batch as one CUDA graph (median of 30), same L2 flush"},
        "reorder_ms_total": reorder_ms,
    }
    if cslt is not None:
        line["cusparselt"] = cslt
    if args.detail and rank == 0:
        for d in detail:
            print(json.dumps(d), file=sys.stderr)
    if rank == 0:
        print(json.dumps(line))
    for h in hs:
        h.free()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
