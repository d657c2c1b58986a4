#!/usr/bin/env python
"""bench.py -- SpMM effective TFLOP/s and speedup vs cuBLAS fp16 GEMM vs sparsity
(BASELINE.json metric) for the Jigsaw hot path on B200.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c2|c1|c3|c4|c5a|c5b|venom]
                  [--impl jigsaw|reference] [--panel-rows 0|128|256] [--no-extra] [--multi]

A STEP is one pass of the SpMM hot path over one batch of synthetic matrices
with the prepared formats resident in HBM (the paper times the kernel only and
excludes format conversion): for the default workload (BASELINE
configs[1], "C2") the batch is the 36 DLMC-transformer-shaped matrices
512x2048 / 2048x512 x v in {2,4,8} x s in {.50,.70,.80,.90,.95,.98}, N = 256,
issued as ONE jigsaw_spmm_batched call (one grouped k_spmm launch).
  value    = sum over the batch of 2*M*N*K (dense-equivalent flops) / step time
  e2e      = the same metric through the C ABI with HOST buffers
             (jigsaw_spmm_batched_host: the batch's B's host->device, grouped
             SpMM, C's device->host, every step)
  e2e_full = + the reorder of A from host memory (jigsaw_reorder_host) every
             step, i.e. every §8(a) row of the hot path
  cublas   = the same products as dense fp16 GEMMs in cuBLAS (the paper's
             baseline): per matrix (cublasGemmEx, best of COMPUTE_16F and
             COMPUTE_32F, L2 flushed before every call) and as a batch (one
             cublasGemmStridedBatchedEx per shape group, best of 16F / 32F,
             timed exactly like the jigsaw step)
  c4       = (default run) the same measurements for BASELINE configs[3], the
             compute-bound Llama-shaped batch, with its tensor roofline
  c5a/c5b  = (N > 1, or --multi) the sharded sweep of configs[4]: 64 DLMC
             matrices split by matrix (LPT), and 4096^2 N = 16384 split by C
             columns; C5b's shards are gathered with NCCL after the timed
             region and checked, and the ranks' format hashes compared
L2 is flushed (256 MB write) before every timed step, outside the events;
per-step device time is taken with CUDA events on the launching stream around
a CUDA-graph replay of the step; multi-GPU: one process per GPU (torchrun),
barrier + synchronize around the timed region, max over ranks.
"""
from __future__ import annotations

import argparse
import json
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
# The paper's own speedups over cuBLAS HGemm (average / max over the DLMC
# matrices), NVIDIA A100 40 GB, fp16 -- PAPER.md Table 2, quoted as
# context only (other GPU, other matrices, other baseline build).
PAPER_TABLE2 = {
    "source": "PAPER.md Table 2 (P:244-259): Jigsaw vs cuBLAS HGemm, A100 40 GB, DLMC, fp16 (avg, max)",
    "v2_s80": [0.77, 1.27], "v4_s80": [0.89, 1.34], "v8_s80": [1.00, 1.67],
    "v2_s90": [1.00, 1.58], "v4_s90": [1.13, 1.95], "v8_s90": [1.35, 1.85],
    "v2_s95": [1.19, 1.73], "v4_s95": [1.44, 2.83], "v8_s95": [1.78, 4.12],
    "v2_s98": [1.43, 1.89], "v4_s98": [1.72, 4.14], "v8_s98": [2.14, 5.45],
}


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
    """HBM GB/s and dense bf16 TF/s (MEASURED_PEAKS.json, driver-written), and the
    measured tcgen05.mma.sp issue-rate peaks (profiles/sparse_mma_peak.json,
    tools/probe_pair_rate.cu on this pool's B200)."""
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        hbm, bf16, src = float(d["hbm_gbs"]), float(d["bf16_tflops"]), "MEASURED_PEAKS.json"
    except Exception:
        hbm, bf16, src = 6650.0, 1590.0, "fallback (B200_PROFILING.md)"
    try:
        sp = json.load(open(os.path.join(ROOT, "profiles", "sparse_mma_peak.json")))
    except Exception:
        sp = {"single_m128_n256_tflops": 2 * bf16, "pair_m256_n256_tflops": 2 * bf16,
              "source": "2 x dense bf16 (no sparse microbenchmark file)"}
    return hbm, bf16, src, sp


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
def algorithmic(info: dict, M: int, K: int, N: int, rows_touched: int, c_bytes_per_elem: int = 2):
    """Per-launch algorithmic bytes and executed flops of k_spmm:
    per tile 16P values + 2P metadata + 64 B gather list, the touched B rows once,
    C once; executed = logical sparse MMA work 2*P*16*N per tile."""
    P = info["panel_rows"]
    a_bytes = (16 * P + 2 * P + 64) * info["ntiles"]
    b_bytes = 2 * N * rows_touched
    c_bytes = c_bytes_per_elem * M * N
    exec_flops = 2 * P * 16 * info["ntiles"] * N
    if info.get("cc_entries"):  # CUDA-core entries (f3): {column, value} 8 B each + per-row offsets
        a_bytes += 8 * info["cc_entries"] + 4 * (info["npanels"] * P + 1)
        exec_flops += 2 * info["cc_entries"] * N
    return a_bytes + b_bytes + c_bytes, exec_flops


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


# ------------------------------------------------------------------ the jigsaw arm
class Batch:
    """One rank's share of a workload, prepared: formats (jigsaw_reorder, untimed,
    P:263), device B / C, host copies of A / B, and the roofline terms."""

    def __init__(self, name, rank, world, panel_rows, dev, torch, jig, cc_max_nnz=0):
        self.name = name
        self.cc_max_nnz = cc_max_nnz
        self.all_points, self.desc, self.scaling = workload(name)
        jobs = local_jobs(name, self.all_points, rank, world)
        self.points = [(M, K, v, s, n1 - n0) for (M, K, v, s, N, seed, n0, n1) in jobs]
        self.jobs = jobs
        self.mats, self.hs, self.dA, self.dB, self.dC = [], [], [], [], []
        self.reorder_ms = 0.0
        self.alg_bytes = self.exec_flops = self.eff_flops = 0
        for ji, (M, K, v, s, N, seed, n0, n1) in enumerate(jobs):
            A = make_a(name, ji, M, K, v, s, seed)
            B = synth.dense_b(K, N, seed)
            if (n0, n1) != (0, N):
                B = np.ascontiguousarray(B[:, n0:n1])
            N = n1 - n0
            self.mats.append((A, B))
            a_t = torch.from_numpy(A.view(np.int16)).to(dev).view(torch.float16)
            h = jig.reorder(a_t, v, panel_rows=panel_rows, cc_max_nnz=cc_max_nnz)
            info = h.info()
            self.reorder_ms += info["reorder_ms"]
            self.hs.append(h)
            self.dA.append(a_t)
            self.dB.append(torch.from_numpy(B.view(np.int16)).to(dev).view(torch.float16))
            self.dC.append(torch.empty((M, N), dtype=torch.float16, device=dev))
            rows_touched = int(((A & 0x7FFF) != 0).any(axis=0).sum())
            ab, ef = algorithmic(info, M, K, N, rows_touched)
            self.alg_bytes += ab
            self.exec_flops += ef
            self.eff_flops += 2 * M * N * K
        self.pair = any(h.info()["panel_rows"] == 256 for h in self.hs)
        self.panel_rows_used = sorted(set(h.info()["panel_rows"] for h in self.hs))

    def step(self, jig):
        jig.spmm_batched(self.hs, self.dB, self.dC)

    def free(self):
        for h in self.hs:
            h.free()


# BENCH_CUDA_PROFILER=1: the first timed region (the headline's K steps) is
# bracketed by cudaProfilerStart/Stop, so `ncu --profile-from-start off` lists
# exactly the launches of the timed steps (tools/gpu_evidence_r02.sh).
_PROFILE_REGION = [os.environ.get("BENCH_CUDA_PROFILER") == "1"]


def timed_steps(fn, steps, warmup, flush, stream, torch, dist=None, world=1, dev_index=0, outside=None):
    """fn captured in a CUDA graph together with two timing events recorded as
    graph nodes immediately before and after it (external event nodes: the
    measured interval is the step's own device work, not the graph launch);
    W warm-up replays, then K replays each preceded by an L2 flush (outside the
    events), barrier + synchronize on both sides of the timed loop, clocks
    sampled during it.  Returns (ms per step, max over ranks; clocks).  If
    `outside` is a dict, it also receives the same steps timed by events around
    the whole graph replay (graph launch latency included)."""
    fn()
    torch.cuda.synchronize()
    e_in0 = torch.cuda.Event(enable_timing=True, external=True)
    e_in1 = torch.cuda.Event(enable_timing=True, external=True)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        e_in0.record()
        fn()
        e_in1.record()
    torch.cuda.synchronize()
    for _ in range(max(3, warmup)):
        flush.zero_()
        g.replay()
    torch.cuda.synchronize()
    sampler = ClockSampler(dev_index)
    sampler.start()
    time.sleep(0.15)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_in, t_out = [], []
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    prof = _PROFILE_REGION[0]
    if prof:
        _PROFILE_REGION[0] = False
        torch.cuda.cudart().cudaProfilerStart()
    for k in range(steps):
        flush.zero_()                     # L2 flush, outside the timed events
        e0.record(stream)
        g.replay()
        e1.record(stream)
        e1.synchronize()                  # the graph's event nodes are re-recorded by the next replay
        t_in.append(e_in0.elapsed_time(e_in1))
        t_out.append(e0.elapsed_time(e1))
    torch.cuda.synchronize()
    if prof:
        torch.cuda.cudart().cudaProfilerStop()
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    from paper_conf_icpp_zhanglyfyllq24_b200 import shard
    dv = torch.device("cuda", dev_index)
    total_ms = shard.max_over_ranks(sum(t_in), dist=dist if world > 1 else None, device=dv)
    if outside is not None:
        outside["ms_per_step"] = shard.max_over_ranks(sum(t_out), dist=dist if world > 1 else None,
                                                      device=dv) / steps
    del g
    return total_ms / steps, clocks


def per_call_us(fn, flush, stream, torch, R=8, reps=7):
    """Device time of one call in a stream of back-to-back kernels, L2 flushed
    before every call: ([graph of R x (flush, call)] - [graph of R x flush]) / R,
    median of `reps` (the event clock moves in ~2 us steps; the difference over
    R calls resolves ~0.1 us)."""
    def graphed(f):
        if f is not None:
            f()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for _ in range(R):
                flush.zero_()
                if f is not None:
                    f()
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
    t0 = timeit(graphed(None))
    return (timeit(graphed(fn)) - t0) / R * 1e3


def roofline(b: Batch, ms_per_step, launches, peaks, traffic_key=None):
    """Roofline of k_spmm (the only kernel of the step, `launches` grouped
    launches of <= 64 products each): algorithmic bytes or executed flops per
    launch over the measured average launch duration (= the step's totals over
    the step time); the binding roof is the larger of bytes / HBM and executed
    flops / the measured tcgen05.mma.sp peak of the variant (CTA pair or single
    CTA)."""
    hbm, bf16, src, sp = peaks
    sp_peak = sp["pair_m256_n256_tflops"] if b.pair else sp["single_m128_n256_tflops"]
    t_hbm = b.alg_bytes / (hbm * 1e9)
    t_tc = b.exec_flops / (sp_peak * 1e12)
    s = ms_per_step * 1e-3
    if t_hbm >= t_tc:
        r = {"bound": "hbm", "achieved": b.alg_bytes / s / 1e9, "peak": hbm, "unit": "GB/s",
             "peak_source": src}
    else:
        r = {"bound": "tensor", "achieved": b.exec_flops / s / 1e12, "peak": sp_peak, "unit": "TFLOP/s",
             "peak_source": f"measured tcgen05.mma.sp {'pair M256' if b.pair else 'M128'} N256 issue rate "
                            f"({sp.get('source', '')}); dense bf16 MEASURED_PEAKS x2 would be {2 * bf16:.0f}"}
    r["frac"] = r["achieved"] / r["peak"]
    r["traffic"] = None
    r["launches_per_step"] = launches
    r["per_launch_us"] = ms_per_step * 1e3 / max(1, launches)
    r["alg_bytes_per_launch"] = b.alg_bytes / max(1, launches)
    r["exec_flops_per_launch"] = b.exec_flops / max(1, launches)
    r["t_roof_us_per_step"] = max(t_hbm, t_tc) * 1e6
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))[traffic_key or b.name]
        r["traffic"] = prof["bytes_per_launch"] if launches == 1 else None
        r["traffic_unit"] = "bytes per launch"
        r["traffic_source"] = prof.get("source")
    except Exception:
        pass
    return r


def cublas_compare(b: Batch, flush, stream, torch, jig, jig_step_ms, steps, warmup, per_matrix=True):
    """cuBLAS dense fp16 GEMM on the dense A of every product (the paper's
    baseline): per matrix best of CUBLAS_COMPUTE_16F / 32F,
    and the batch as one strided-batched GEMM per shape group (best of 16F / 32F),
    timed like the jigsaw step."""
    from tools import cublas_ref
    out = {}
    outs = [torch.empty((M, N), dtype=torch.float16, device=c.device) for c, (M, K, v, s, N) in
            zip(b.dC, b.points)]
    groups = {}
    for i, (M, K, v, s, N) in enumerate(b.points):
        groups.setdefault((M, K, N), []).append(i)
    stk = {}
    for key, idx in groups.items():
        M, K, N = key
        stk[key] = (torch.stack([b.dA[i] for i in idx]), torch.stack([b.dB[i] for i in idx]),
                    torch.empty((len(idx), M, N), dtype=torch.float16, device=b.dA[0].device))
    batched = {}
    for comp in ("16F", "32F"):
        def step(comp=comp):
            for A3, B3, C3 in stk.values():
                cublas_ref.gemm_strided_batched(A3, B3, C3, comp)
        batched[comp], _ = timed_steps(step, steps, warmup, flush, stream, torch)
    best = min(batched, key=batched.get)
    out["batched_step_ms"] = batched[best]
    out["batched_compute"] = best
    out["batched_step_ms_16F_32F"] = [batched["16F"], batched["32F"]]
    out["speedup_vs_batched_cublas"] = batched[best] / jig_step_ms
    if b.name == "venom":
        out["cusparselt"] = cusparselt_compare(b, flush, stream, torch, jig_step_ms, steps, warmup)
    out["batched_how"] = ("one cublasGemmStridedBatchedEx per (M, K, N) group of the batch, best of "
                          "CUBLAS_COMPUTE_16F / 32F, graph-replayed and timed exactly like the jigsaw step "
                          "(event nodes around the step inside its graph, L2 flushed before)")
    if not per_matrix:
        return out
    detail, sp = [], {}
    tj_sum = tc_sum = 0.0
    for i, (M, K, v, s, N) in enumerate(b.points):
        tj = per_call_us(lambda: b.hs[i].spmm(b.dB[i], C=b.dC[i]), flush, stream, torch)
        t16 = per_call_us(lambda: cublas_ref.gemm(b.dA[i], b.dB[i], outs[i], "16F"), flush, stream, torch)
        t32 = per_call_us(lambda: cublas_ref.gemm(b.dA[i], b.dB[i], outs[i], "32F"), flush, stream, torch)
        tc = min(t16, t32)
        tag = point_tag(b.name, i, v, s)
        detail.append({"M": M, "K": K, "v": v, "s": s, "N": N, "tag": tag, "jigsaw_us": tj,
                       "cublas16F_us": t16, "cublas32F_us": t32, "speedup": tc / tj,
                       "eff_tflops": 2 * M * N * K / (tj * 1e-6) / 1e12})
        sp.setdefault(tag, []).append(tc / tj)
        tj_sum += tj
        tc_sum += tc
    out["speedup_geomean_by_v_s"] = {k: float(np.exp(np.mean(np.log(x)))) for k, x in sorted(sp.items())}
    out["paper_context"] = PAPER_TABLE2
    out["per_matrix_speedup_total_time"] = tc_sum / tj_sum
    out["per_matrix_how"] = ("each product alone: jigsaw_spmm vs cublasGemmEx (best of COMPUTE_16F / 32F) on "
                             "the dense A, [graph of 8 x (L2 flush, call)] - [graph of 8 x flush], / 8, median of 7")
    out["detail"] = detail
    return out


def cusparselt_compare(b: Batch, flush, stream, torch, jig_step_ms, steps, warmup):
    """f4 (Table 3): the library 2:4 SpMM (cuSPARSELt via
    torch._cslt_compress / torch._cslt_sparse_mm) on the natively 2:4 VENOM-style
    A -- it cannot skip the all-zero columns Jigsaw's reorder removes -- per
    matrix and as a batch, timed like the jigsaw step."""
    try:
        comp = [torch._cslt_compress(a) for a in b.dA]
        torch._cslt_sparse_mm(comp[0], b.dB[0])
        torch.cuda.synchronize()
    except Exception as e:  # library without an sm_100 build, or API absent
        return {"unavailable": f"{type(e).__name__}: {str(e).splitlines()[0][:200]}"}
    outs = [None] * len(comp)

    def step():
        for i, (a, bb) in enumerate(zip(comp, b.dB)):
            outs[i] = torch._cslt_sparse_mm(a, bb)
    ms, _ = timed_steps(step, steps, warmup, flush, stream, torch)
    per = {}
    for i, (M, K, v, s, N) in enumerate(b.points):
        tj = per_call_us(lambda: b.hs[i].spmm(b.dB[i], C=b.dC[i]), flush, stream, torch)
        tc = per_call_us(lambda: torch._cslt_sparse_mm(comp[i], b.dB[i]), flush, stream, torch)
        per.setdefault(point_tag(b.name, i, v, s), []).append(tc / tj)
    return {"step_ms": ms, "speedup_step": ms / jig_step_ms,
            "speedup_geomean_by_point": {k: float(np.exp(np.mean(np.log(x)))) for k, x in sorted(per.items())},
            "how": "torch._cslt_compress / torch._cslt_sparse_mm (cuSPARSELt 2:4 SpMM) on the natively 2:4 A; "
                   "batch = one graph of the per-matrix calls timed like the jigsaw step, per matrix = graph "
                   "difference with L2 flushed"}


def e2e_host(b: Batch, jig, torch, steps, dist=None, world=1, dev=None, warmup=3):
    """The metric end to end through the public API with HOST buffers
    (jigsaw_spmm_batched_host: pinned B's in, grouped SpMM, C's out, every step).
    Host-side copy times vary from step to step on these boxes (C4: 7.2-14.7 ms
    per step in one process, profiles/r02at_e2e_pack.jsonl), so `warmup` untimed
    calls precede the timed ones."""
    # the batch's B's in one pinned block and its C's in another (views, back to
    # back): jigsaw_spmm_batched_host then moves each chunk with one copy per
    # direction instead of one per product
    nb = sum(B.size for (_, B) in b.mats)
    nc = sum(M * N for (M, K, v, s, N) in b.points)
    blk_b = torch.empty(nb, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
    blk_c = torch.empty(nc, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
    pin_B, pin_C, ob, oc = [], [], 0, 0
    for (_, B), (M, K, v, s, N) in zip(b.mats, b.points):
        pin_B.append(blk_b[ob:ob + B.size].reshape(B.shape))
        pin_B[-1][...] = B
        pin_C.append(blk_c[oc:oc + M * N].reshape(M, N))
        ob += B.size
        oc += M * N
    h2d = sum(B.nbytes for (_, B) in b.mats)
    d2h = sum(2 * M * N for (M, K, v, s, N) in b.points)
    for _ in range(max(1, warmup)):
        jig.spmm_batched_host(b.hs, pin_B, pin_C)
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(steps):
        jig.spmm_batched_host(b.hs, pin_B, pin_C)
    e2e_s = (time.perf_counter() - t0) / steps
    from paper_conf_icpp_zhanglyfyllq24_b200 import shard
    e2e_s = shard.max_over_ranks(e2e_s, dist=dist if world > 1 else None, device=dev)
    return e2e_s, h2d, d2h


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--panel-rows", type=int, default=0, choices=[0, 128, 256],
                    help="reorder panel height: 0 = library auto, 128 (one CTA per panel) or 256 (CTA pairs)")
    ap.add_argument("--impl", default="jigsaw", choices=["jigsaw", "reference"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-cublas", action="store_true")
    ap.add_argument("--no-extra", action="store_true", help="skip the c4 sub-object of the default run")
    ap.add_argument("--multi", action="store_true", help="also run the C5a / C5b sharded sweep at N = 1")
    ap.add_argument("--detail", action="store_true", help="print the per-point table to stderr")
    ap.add_argument("--cc-max-nnz", type=int, default=0,
                    help="CUDA-core tiles (f3, R-Q28): tiles with <= Z nonzeros run on CUDA cores (0 = none)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        os.environ.setdefault("NCCL_DEBUG", "INFO")          # communicator init (nranks) in the log
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    import torch
    import torch.distributed as dist
    import paper_conf_icpp_zhanglyfyllq24_b200 as jig

    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        print(f"[bench] rank {rank}: NCCL process group up, world size {dist.get_world_size()}", file=sys.stderr)
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    stream = torch.cuda.current_stream()
    peaks = load_peaks()
    flush = torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev)
    dist_ = dist if world > 1 else None

    b = Batch(args.workload, rank, world, args.panel_rows, dev, torch, jig, cc_max_nnz=args.cc_max_nnz)
    total_eff = sum(2 * M * K * N for (M, K, v, s, N) in b.all_points) * (world if b.scaling == "weak" else 1)
    b.step(jig)
    torch.cuda.synchronize()
    launches = jig.last_launch()["launches"]
    outside = {}
    ms, clocks = timed_steps(lambda: b.step(jig), args.steps, args.warmup, flush, stream, torch,
                             dist=dist_, world=world, dev_index=dev.index or 0, outside=outside)
    value = total_eff / (ms * 1e-3) / 1e12
    roof = roofline(b, ms, launches, peaks)

    cub = None
    if not args.no_cublas and b.points:
        cub = cublas_compare(b, flush, stream, torch, jig, ms, min(args.steps, 30), args.warmup)
        if args.detail and rank == 0:
            for d in cub["detail"]:
                print(json.dumps(d), file=sys.stderr)
        cub.pop("detail", None)

    e2e_steps = max(3, min(args.steps, 20))
    e2e_s, h2d, d2h = e2e_host(b, jig, torch, e2e_steps, dist_, world, dev)
    # e2e_full: host A -> reorder -> host B -> SpMM -> host C (all §8(a) rows), rank 0 batch, one pass
    t0 = time.perf_counter()
    for (A, B), (M, K, v, s, N) in zip(b.mats, b.points):
        hh = jig.reorder_host(A, v, panel_rows=args.panel_rows)
        hh.spmm_host(B)
        hh.free()
    full_s = time.perf_counter() - t0

    line = {
        "metric": METRIC, "value": value, "unit": "TFLOP/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
        "higher_is_better": True, "scaling": b.scaling, "vs_baseline": None, "dtype": "f16",
        "data": "synthetic",
        "config": {"workload": b.desc, "matrices_on_rank0": len(b.points),
                   "flops": "dense-equivalent 2*M*N*K per matrix",
                   "l2": "flushed (256 MB write) before every timed step",
                   "launch": "step = one jigsaw_spmm_batched call over the batch (one grouped k_spmm launch per "
                             "64 matrices of one panel height), captured in a CUDA graph",
                   "timing": "CUDA events recorded as nodes of the step's graph around the k_spmm launch "
                             "(stream of the launch); events around the whole graph replay, graph launch latency "
                             f"included: {outside.get('ms_per_step', 0) * 1e3:.1f} us per step",
                   "seeds": "synth.SEED_BASE + 1000*rank + index",
                   "format": f"panel_rows={args.panel_rows or 'auto'} (P used: {b.panel_rows_used}), SPTC residual"
                             + (f", cc_max_nnz={args.cc_max_nnz}" if args.cc_max_nnz else "")},
        "roofline": roof,
        "cpu_baseline": None,
        "e2e": {"value": total_eff / e2e_s / 1e12, "unit": "TFLOP/s",
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "ms_per_step": e2e_s * 1e3, "steps": e2e_steps,
                "call": "jigsaw_spmm_batched_host (the batch's B's and C's packed in one pinned block each), "
                        "wall clock per step after 3 untimed calls, max over ranks"},
        "e2e_full": {"value": b.eff_flops / full_s / 1e12, "unit": "TFLOP/s",
                     "note": "this rank: jigsaw_reorder_host + jigsaw_spmm_host per matrix, one pass"},
        "gpu_launches": launches * args.steps,
        "clocks": clocks,
        "cublas": cub,
        "reorder_ms_total": b.reorder_ms,
    }

    # ---- C4 (configs[3]) alongside the default C2 line: compute-bound, CTA pairs
    if args.workload == "c2" and not args.no_extra:
        b4 = Batch("c4", rank, world, 0, dev, torch, jig)
        b4.step(jig)
        torch.cuda.synchronize()
        l4 = jig.last_launch()["launches"]
        st4 = max(5, min(args.steps, 20))
        ms4, clk4 = timed_steps(lambda: b4.step(jig), st4, args.warmup, flush, stream, torch,
                                dist=dist_, world=world, dev_index=dev.index or 0)
        eff4 = sum(2 * M * K * N for (M, K, v, s, N) in b4.all_points) * world
        c4 = {"workload": b4.desc, "value": eff4 / (ms4 * 1e-3) / 1e12, "unit": "TFLOP/s", "ms_per_step": ms4,
              "steps": st4, "gpu_launches": l4 * st4, "roofline": roofline(b4, ms4, l4, peaks),
              "clocks": clk4, "format": f"panel_rows=auto (P used: {b4.panel_rows_used})",
              "reorder_ms_total": b4.reorder_ms}
        if not args.no_cublas:
            cb4 = cublas_compare(b4, flush, stream, torch, jig, ms4, st4, args.warmup)
            cb4.pop("detail", None)
            c4["cublas"] = cb4
        e4, h4, d4 = e2e_host(b4, jig, torch, 12, dist_, world, dev)
        c4["e2e"] = {"value": eff4 / e4 / 1e12, "unit": "TFLOP/s", "h2d_bytes_per_step": h4,
                     "d2h_bytes_per_step": d4, "ms_per_step": e4 * 1e3, "steps": 12}
        line["c4"] = c4
        b4.free()

    # ---- C5a / C5b (configs[4]): the sharded sweep, at N > 1 (or --multi)
    if (world > 1 or args.multi) and args.workload == "c2":
        from paper_conf_icpp_zhanglyfyllq24_b200 import shard
        for name in ("c5a", "c5b"):
            bs = Batch(name, rank, world, 0, dev, torch, jig)
            st5 = max(5, min(args.steps, 20))
            fn = (lambda: bs.step(jig)) if bs.hs else (lambda: None)
            ms5, clk5 = timed_steps(fn, st5, args.warmup, flush, stream, torch,
                                    dist=dist_, world=world, dev_index=dev.index or 0)
            eff5 = sum(2 * M * K * N for (M, K, v, s, N) in bs.all_points)
            sub = {"workload": bs.desc, "value": eff5 / (ms5 * 1e-3) / 1e12, "unit": "TFLOP/s",
                   "ms_per_step": ms5, "steps": st5, "scaling": "strong", "matrices_on_rank0": len(bs.points),
                   "clocks": clk5}
            if name == "c5b" and world >= 1:
                # untimed validation: NCCL all_gather of the C column shards, sampled
                # rows checked on rank 0 against a dense PyTorch product; the ranks'
                # format hashes (deterministic reorder of the replicated A) compared
                M, K, v, s, N, seed, n0, n1 = local_jobs("c5b", bs.all_points, rank, world)[0]
                torch.cuda.synchronize()
                full = shard.gather_column_shards(bs.dC[0], n0, n1, N, dist, world) if world > 1 else bs.dC[0]
                hsh = torch.tensor([shard.format_hash(bs.hs[0].export())], dtype=torch.int64, device=dev)
                hs_all = [torch.zeros_like(hsh) for _ in range(world)]
                if world > 1:
                    dist.all_gather(hs_all, hsh)
                else:
                    hs_all = [hsh]
                if rank == 0:
                    Bfull = torch.from_numpy(synth.dense_b(K, N, seed).view(np.int16)).to(dev).view(torch.float16)
                    rows = torch.from_numpy(np.sort(np.random.default_rng(5).choice(M, 64, replace=False))).to(dev)
                    excess = shard.check_against_dense(full, bs.dA[0], Bfull, rows)
                    sub["validation"] = {"gathered_shape": list(full.shape), "rows_checked": 64,
                                         "max_excess_over_tolerance": excess, "pass": excess <= 0,
                                         "format_hashes_equal": len({int(x.item()) for x in hs_all}) == 1,
                                         "how": "all_gather of C column shards (NCCL) after the timed region; "
                                                "64 sampled rows vs torch fp32 matmul of the dense fp16 A"}
            line[name] = sub
            bs.free()

    if rank == 0 and world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(b.points, b.mats)
    if rank == 0:
        print(json.dumps(line))
    b.free()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
