"""Multi-GPU partitioning of the hot path.

The SpMM partitions into independent work with no exchange on the data path:
  * column shards of B / C (C5b): rank g computes C[:, n0:n1] = A . B[:, n0:n1]
    with the (deterministically rebuilt) format of A replicated on every rank;
  * independent matrices (C5a): greedy LPT assignment by estimated cost.
NCCL (torch.distributed) only carries barriers, the max-over-ranks timing and
the untimed validation gather.  Pure host logic; covered by
tests/test_dist_gloo.py on CPU with world size 2.
"""
from __future__ import annotations


def column_shards(N: int, world: int, align: int = 128):
    """Split columns [0, N) into `world` contiguous shards whose boundaries are
    multiples of `align` (a 128-column C tile never straddles two ranks).
    Returns [(n0, n1)] per rank; shards may be empty when N is small."""
    if N <= 0 or world <= 0 or align <= 0:
        raise ValueError("N, world and align must be positive")
    tiles = -(-N // align)
    out, t0 = [], 0
    for g in range(world):
        t1 = t0 + tiles // world + (1 if g < tiles % world else 0)
        out.append((min(N, t0 * align), min(N, t1 * align)))
        t0 = t1
    return out


def lpt_assign(costs, world: int):
    """Longest-processing-time-first greedy assignment of independent jobs.
    Returns a list of job-index lists, one per rank (deterministic)."""
    loads = [0.0] * world
    bins = [[] for _ in range(world)]
    for j in sorted(range(len(costs)), key=lambda j: (-costs[j], j)):
        g = min(range(world), key=lambda g: (loads[g], g))
        bins[g].append(j)
        loads[g] += costs[j]
    return [sorted(b) for b in bins]


def spmm_cost(info: dict, N: int) -> float:
    """Estimated device work of one product: executed sparse MMA work plus bytes."""
    P = info["panel_rows"]
    return 2.0 * P * 16 * info["ntiles"] * N / 3.0e15 + (18 * P + 64) * info["ntiles"] / 6.0e12


def max_over_ranks(x: float, dist=None, device=None) -> float:
    """Max of a scalar over all ranks (identity without a process group)."""
    if dist is None or not dist.is_available() or not dist.is_initialized():
        return x
    import torch
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_column_shards(C_local, n0: int, n1: int, N: int, dist, world: int):
    """Validation gather (untimed; north_star "NCCL only to gather C for
    validation"): every rank contributes its column shard C[:, n0:n1] (padded to
    the widest shard, so the collective moves equal-size buffers); returns the
    assembled M x N tensor on every rank.  Works on any backend (NCCL on GPUs,
    gloo in the CPU tests)."""
    import torch
    M = C_local.shape[0]
    shards = column_shards(N, world)
    width = max(b - a for a, b in shards)
    pad = torch.zeros((M, width), dtype=C_local.dtype, device=C_local.device)
    pad[:, : n1 - n0] = C_local
    parts = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(parts, pad)
    return torch.cat([p[:, : b - a] for p, (a, b) in zip(parts, shards)], dim=1)


def format_hash(arrays: dict) -> int:
    """64-bit hash (BLAKE2b) of a canonical format (jigsaw_export_format arrays,
    fixed key order): ranks that rebuilt the replicated A must agree."""
    import hashlib

    import numpy as np
    h = hashlib.blake2b(digest_size=8)
    for k in sorted(arrays):
        h.update(k.encode())
        h.update(np.ascontiguousarray(arrays[k]).tobytes())
    return int.from_bytes(h.digest(), "little") & 0x7FFFFFFFFFFFFFFF


def check_against_dense(C, A_dense, B, rows, tol_rel: float = 1e-2, tol_abs: float = 1e-3):
    """Sampled-row check of a (gathered) C against a plain dense PyTorch product
    of the same fp16 inputs in fp32 (no oracle on the benchmark path): |C - A.B|
    <= tol_rel (|A|.|B|) + tol_abs, the north_star tolerance.  Returns the max
    excess (<= 0 means pass)."""
    import torch
    a = A_dense[rows].float()
    ref = a @ B.float()
    mabs = a.abs() @ B.float().abs()
    err = (C[rows].float() - ref).abs()
    return float((err - (tol_rel * mabs + tol_abs)).max())
