"""Multi-process (gloo, world size 2, CPU) coverage of the N > 1 path: column
sharding of B/C and LPT assignment of independent matrices, the max-over-ranks
timing, and the (untimed) validation gather -- with the oracle standing in for
the per-rank GPU product (no GPU here)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_zhanglyfyllq24_b200 import shard


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import synth
        M, K, N = 256, 192, 384
        A = synth.vector_sparse(M, K, 8, 0.9, 1)           # same seed on every rank (replicated A)
        B = synth.dense_b(K, N, 1)
        n0, n1 = shard.column_shards(N, world)[rank]
        Cs, _ = oracle.spmm(A, np.ascontiguousarray(B[:, n0:n1]))
        # validation gather (untimed in bench.py): every rank contributes its columns
        parts = [None] * world
        dist.all_gather_object(parts, (n0, n1, Cs))
        full = np.zeros((M, N))
        for a, b, c in parts:
            full[:, a:b] = c
        ref, _ = oracle.spmm(A, B)
        ok_cols = np.array_equal(full, ref)
        # format hash agreement: every rank rebuilds the same CR1 format
        f = oracle.reorder(A, P=128)
        hsh = torch.tensor([int(f.meta.sum()) + 7 * int(f.col_idx.sum())], dtype=torch.int64)
        hs = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(hs, hsh)
        ok_hash = all(int(h) == int(hsh) for h in hs)
        mx = shard.max_over_ranks(float(rank + 1), dist=dist, device="cpu")
        # the helpers bench.py uses after the timed region (NCCL on GPUs): padded
        # shard gather, format hash, sampled-row check against a dense product
        Ct = torch.from_numpy(Cs.astype(np.float32))
        full_t = shard.gather_column_shards(Ct, n0, n1, N, dist, world)
        ok_gather = np.array_equal(full_t.numpy().astype(np.float64), full.astype(np.float32).astype(np.float64))
        fh = shard.format_hash({"T": f.T, "meta": f.meta, "col_idx": f.col_idx})
        hs2 = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(hs2, torch.tensor([fh], dtype=torch.int64))
        ok_fh = len({int(h) for h in hs2}) == 1
        Ad = torch.from_numpy(A.view(np.float16).astype(np.float32))
        Bd = torch.from_numpy(B.view(np.float16).astype(np.float32))
        excess = shard.check_against_dense(full_t, Ad, Bd, torch.arange(0, M, 7))
        bad = full_t.clone()
        bad[5, 3] += 1.0
        excess_bad = shard.check_against_dense(bad, Ad, Bd, torch.tensor([5]))
        q.put((rank, ok_cols and ok_gather and ok_fh and excess <= 0 and excess_bad > 0, ok_hash, mx))
    finally:
        dist.destroy_process_group()


def test_two_rank_column_shards_gloo():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    res = sorted(q.get(timeout=10) for _ in range(world))
    for rank, ok_cols, ok_hash, mx in res:
        assert ok_cols and ok_hash and mx == float(world)


def test_column_shards_cover_exactly_once():
    for N in [8, 128, 136, 256, 1000, 16384]:
        for world in [1, 2, 3, 4, 8]:
            sh = shard.column_shards(N, world)
            assert len(sh) == world
            cols = np.concatenate([np.arange(a, b) for a, b in sh])
            assert np.array_equal(cols, np.arange(N))
            assert all(a % 128 == 0 for a, b in sh if b > a)


def test_lpt_assign_balanced_and_complete():
    rng = np.random.default_rng(0)
    costs = list(rng.uniform(1, 10, size=64))
    bins = shard.lpt_assign(costs, 8)
    assert sorted(j for b in bins for j in b) == list(range(64))
    loads = [sum(costs[j] for j in b) for b in bins]
    assert max(loads) <= sum(costs) / 8 + max(costs)
    assert shard.lpt_assign(costs, 8) == bins       # deterministic
