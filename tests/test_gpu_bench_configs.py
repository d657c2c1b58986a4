"""GPU parity of the exact configurations bench.py times, of the fp32-C option
and of concurrent launches (CUDA-graph replays on several streams).

  * C2 (BASELINE configs[1]): the 36-matrix batch with bench.py's seeds through
    ONE jigsaw_spmm_batched call -- the same grouped launch (tile width,
    dynamic scheduler, pieces) the timed step replays -- every matrix against
    the oracle on sampled rows + the last rows, format bit-exact on a sampled
    panel, and the integer-valued twin of the batch bit-exact (fp32 C);
  * C4 (configs[3]): the 8 Llama-shaped matrices at the auto panel height
    (256-row panels on CTA pairs), N = 2048, the launch bench.py times;
  * c_dtype = JIGSAW_C_F32 on every launch shape;
  * graphs captured from jigsaw_spmm_batched replayed concurrently on two
    streams, next to eager calls on a third, many times (launch-tagged
    counters, graph-owned workspaces).
Tolerance: |C - C_ref| <= 1e-2 (|A|.|B|) + 1e-3 (north_star); integers exact.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import bench  # noqa: E402  (bench.py's workload definitions and seeds)
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402
from test_gpu_parity import _dev, _host, assert_format_equal, int_exact, spmm_check  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.set_device(0)


def _rows(M, n, seed):
    rng = np.random.default_rng(seed)
    r = rng.choice(M, size=min(n, M), replace=False)
    return np.unique(np.concatenate([r, np.arange(max(0, M - 8), M)]))


def _batch(workload, kind="uniform", c_dtype=0, panel_rows=0):
    pts, _, _ = bench.workload(workload)
    mats, hs, dB, dC = [], [], [], []
    for i, (M, K, v, s, N) in enumerate(pts):
        seed = bench.point_seed(i, 0)
        A = bench.make_a(workload, i, M, K, v, s, seed) if kind == "uniform" else \
            synth.vector_sparse(M, K, v, s, seed, kind="int")
        B = synth.dense_b(K, N, seed, kind=kind)
        mats.append((A, B, v))
        hs.append(jig.reorder(_dev(A), v, panel_rows=panel_rows, c_dtype=c_dtype))
        dB.append(_dev(B))
        dC.append(torch.full((M, N), 7.0, dtype=torch.float32 if c_dtype else torch.float16, device="cuda"))
    return pts, mats, hs, dB, dC


def test_bench_c2_batch():
    """C2 exactly as timed: 36 matrices, bench.py seeds, one grouped launch."""
    pts, mats, hs, dB, dC = _batch("c2")
    jig.spmm_batched(hs, dB, dC)
    torch.cuda.synchronize()
    d = jig.last_launch()
    assert d["launches"] == 1 and d["problems"] == 36 and d["cta_pair"] == 0, d
    assert d["dynamic_schedule"] == 0 and d["work_items"] >= 720, d     # the host's static LPT plan
    for i, ((A, B, v), c) in enumerate(zip(mats, dC)):
        M = A.shape[0]
        spmm_check(_host(c), A, B, rows=_rows(M, 64, i))
        p = (i * 7) % ((M + 127) // 128)
        assert_format_equal(hs[i].export(), oracle.reorder(A, P=128, panels=(p, p + 1)), panels=(p, p + 1))
    # graph replay of the same call (the bench's timed form), outputs refilled
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        jig.spmm_batched(hs, dB, dC)
    for c in dC:
        c.fill_(3.0)
    g.replay()
    torch.cuda.synchronize()
    for i, ((A, B, v), c) in enumerate(zip(mats, dC)):
        spmm_check(_host(c), A, B, rows=_rows(A.shape[0], 16, 100 + i))


def test_bench_c2_batch_integer_exact():
    """The integer-valued twin of the C2 batch (same shapes, sparsities, seeds;
    A in {+-1,+-2}, B in {-2..2}) with fp32 C: bit-exact on 128 sampled rows of
    every matrix."""
    pts, mats, hs, dB, dC = _batch("c2", kind="int", c_dtype=jig.C_F32)
    jig.spmm_batched(hs, dB, dC)
    torch.cuda.synchronize()
    for i, ((A, B, v), c) in enumerate(zip(mats, dC)):
        int_exact(_host(c), A, B, rows=_rows(A.shape[0], 128, 200 + i))


def test_bench_c4_batch():
    """C4 exactly as timed: 8 Llama-shaped matrices, v = 8, N = 2048, auto panel
    height (256-row panels, CTA pairs), one grouped launch; 40 sampled rows +
    the last rows per matrix, a sampled panel bit-exact."""
    pts, mats, hs, dB, dC = _batch("c4")
    jig.spmm_batched(hs, dB, dC)
    torch.cuda.synchronize()
    d = jig.last_launch()
    assert d["launches"] == 1 and d["problems"] == 8 and d["cta_pair"] == 1, d
    for i, ((A, B, v), c) in enumerate(zip(mats, dC)):
        M = A.shape[0]
        assert hs[i].info()["panel_rows"] == 256
        spmm_check(_host(c), A, B, rows=_rows(M, 40, 300 + i))
    A = mats[1][0]
    assert_format_equal(hs[1].export(), oracle.reorder(A, P=256, panels=(5, 6)), panels=(5, 6))


@pytest.mark.parametrize("shape", ["split", "nt32", "single128", "grouped_pieces", "grouped_nsplit", "pair",
                                   "pair_nsplit"])
def test_c_dtype_f32(shape):
    """jigsaw_options_t.c_dtype = JIGSAW_C_F32: C is the fp32 accumulator (R-Q17),
    on every launch shape; float inputs within tolerance, integer inputs bit-exact
    with no range limit below 2^24."""
    P, ov, M, K, v, s, N = 128, {}, 512, 1024, 4, 0.8, 256
    if shape == "split":
        ov = dict(split_k=4)
    elif shape == "nt32":
        ov = dict(tile_n=32, split_k=2)
        N = 200
    elif shape == "single128":
        ov = dict(tile_n=128)
        M, N = 640, 328
    elif shape == "pair":
        P, M, N = 256, 600, 264
    elif shape == "grouped_pieces":
        ov = dict(k_pieces=1)
    A = synth.vector_sparse(M, K, v, s, 51)
    B = synth.dense_b(K, N, 51)
    Ai = synth.vector_sparse(M, K, v, s, 52, kind="int")
    Bi = synth.dense_b(K, N, 52, kind="int")
    with jig.launch_override(**ov):
        if shape in ("grouped_pieces", "grouped_nsplit", "pair_nsplit"):
            Pg = 256 if shape == "pair_nsplit" else 128
            big = synth.vector_sparse(512, 6000, 2, 0.5, 53, kind="int")
            bigB = synth.dense_b(6000, 256, 54, kind="int")
            hs = [jig.reorder(_dev(big), 2, panel_rows=Pg, c_dtype=jig.C_F32)] + \
                 [jig.reorder(_dev(synth.vector_sparse(128, 96, 4, 0.8, 60 + j, kind="int")), 4, panel_rows=Pg,
                              c_dtype=jig.C_F32) for j in range(12)]
            Bs = [bigB] + [synth.dense_b(96, 64, 70 + j, kind="int") for j in range(12)]
            mats = [big] + [synth.vector_sparse(128, 96, 4, 0.8, 60 + j, kind="int") for j in range(12)]
            dC = [torch.empty((h.M, b.shape[1]), dtype=torch.float32, device="cuda") for h, b in zip(hs, Bs)]
            jig.spmm_batched(hs, [_dev(b) for b in Bs], dC)
            torch.cuda.synchronize()
            d = jig.last_launch()
            assert (d["split_slots"] > 0) if shape == "grouped_pieces" else (d["nsplit_items"] > 0), d
            for a, b, c in zip(mats, Bs, dC):
                int_exact(_host(c), a, b)
            return
        h = jig.reorder(_dev(A), v, panel_rows=P, c_dtype=jig.C_F32)
        assert h.info()["c_dtype"] == jig.C_F32
        C = h.spmm(_dev(B))
        assert C.dtype == torch.float32
        hi = jig.reorder(_dev(Ai), v, panel_rows=P, c_dtype=jig.C_F32)
        Ci = hi.spmm(_dev(Bi))
        torch.cuda.synchronize()
    spmm_check(_host(C), A, B)
    int_exact(_host(Ci), Ai, Bi)
    # host-buffer paths with fp32 C
    Ch = h.spmm_host(B)
    assert Ch.dtype == np.float32
    spmm_check(Ch, A, B)
    outs = jig.spmm_batched_host([h, hi], [B, Bi])
    spmm_check(outs[0], A, B)
    int_exact(outs[1], Ai, Bi)


def _int_batch(n_small=10, seed0=800):
    mats = [synth.vector_sparse(512, 6000, 2, 0.5, seed0, kind="int")]
    Bs = [synth.dense_b(6000, 200, seed0 + 1, kind="int")]
    for i in range(n_small):
        mats.append(synth.vector_sparse(256, 640, 4, 0.8, seed0 + 10 + i, kind="int"))
        Bs.append(synth.dense_b(640, 136, seed0 + 30 + i, kind="int"))
    hs = [jig.reorder(_dev(a), 2 if i == 0 else 4) for i, a in enumerate(mats)]
    refs = [oracle.spmm(a, b)[0] for a, b in zip(mats, Bs)]
    assert max(np.abs(r).max() for r in refs) <= 2048, "integer fixture must stay exact in fp16"
    return mats, Bs, hs, refs


def test_graph_replays_concurrent_streams():
    """Two CUDA graphs captured from jigsaw_spmm_batched (dynamic scheduler + k-range
    pieces, each with its graph-owned workspace), replayed concurrently on two
    streams 6 times each while eager calls of the same batch run on a third
    stream (its own per-stream workspace); every output bit-exact (integer
    inputs).  Before the workspace became per stream / per captured launch,
    concurrent launches could share a scheduler counter and partial tiles."""
    mats, Bs, hs, refs = _int_batch()
    dB = [_dev(b) for b in Bs]
    outs = [[torch.empty((a.shape[0], b.shape[1]), dtype=torch.float16, device="cuda") for a, b in zip(mats, Bs)]
            for _ in range(3)]
    graphs = []
    jig.set_launch_override(k_pieces=1)          # k-range pieces: the workspace-heavy path
    for k in range(2):
        jig.spmm_batched(hs, dB, outs[k])   # warm-up outside capture
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            jig.spmm_batched(hs, dB, outs[k])
        d = jig.last_launch()
        assert d["graph_owned_workspace"] == 1 and d["split_slots"] > 0, d
        graphs.append(g)
    streams = [torch.cuda.Stream() for _ in range(3)]
    big = torch.randn(4096, 4096, device="cuda", dtype=torch.float16)
    torch.cuda.synchronize()
    try:
        _run_concurrent(graphs, streams, big, outs, hs, dB, refs)
    finally:
        jig.set_launch_override()


def _run_concurrent(graphs, streams, big, outs, hs, dB, refs):
    for rep in range(6):
        for k, st in enumerate(streams):
            with torch.cuda.stream(st):
                _ = big @ big                  # queue the three streams behind long kernels ...
                for c in outs[k]:
                    c.fill_(5.0)
        for k, st in enumerate(streams):       # ... so the SpMMs below run at the same time
            with torch.cuda.stream(st):
                if k < 2:
                    graphs[k].replay()
                else:
                    jig.spmm_batched(hs, dB, outs[2], stream=st)
        torch.cuda.synchronize()
        for k in range(3):
            for r, c in zip(refs, outs[k]):
                assert np.array_equal(_host(c).view(np.float16).astype(np.float64), r), (rep, k)


def test_many_replays_counters():
    """One captured batch replayed 40 times back to back (no host sync between
    replays): every replay zeroes its graph-owned counters (memset node) and
    must schedule every unit and reduce every split unit exactly once; then the
    same batch 40 times eagerly on one stream (per-stream workspace whose
    counters each launch leaves at zero)."""
    mats, Bs, hs, refs = _int_batch(n_small=6, seed0=900)
    dB = [_dev(b) for b in Bs]
    jig.set_launch_override(k_pieces=1)
    dC = [torch.empty((a.shape[0], b.shape[1]), dtype=torch.float16, device="cuda") for a, b in zip(mats, Bs)]
    acc = [torch.zeros((a.shape[0], b.shape[1]), dtype=torch.float32, device="cuda") for a, b in zip(mats, Bs)]
    jig.spmm_batched(hs, dB, dC)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for c in dC:
            c.fill_(9.0)
        jig.spmm_batched(hs, dB, dC)
        for a_, c in zip(acc, dC):
            a_.add_(c.float())
    for _ in range(40):
        g.replay()
    torch.cuda.synchronize()
    for r, a_ in zip(refs, acc):
        assert np.array_equal(a_.cpu().numpy().astype(np.float64), 40.0 * r)
    jig.set_launch_override()
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        for a_ in acc:
            a_.zero_()
        for _ in range(40):
            jig.spmm_batched(hs, dB, dC, stream=st)
            for a_, c in zip(acc, dC):
                a_.add_(c.float())
    torch.cuda.synchronize()
    for r, a_ in zip(refs, acc):
        assert np.array_equal(a_.cpu().numpy().astype(np.float64), 40.0 * r)


def test_single_product_dynamic_scheduler():
    """A single product with more 64-column units than CTAs and no host plan runs
    the dynamic tile scheduler (ticket in the per-stream workspace, reset by the
    last CTA): eager calls on two streams and replays of a captured graph, all
    bit-exact on integer inputs."""
    M, K, N = 12800, 96, 128          # 100 panels: 100 units of 128 columns, 200 of 64
    A = synth.vector_sparse(M, K, 4, 0.8, 901, kind="int")
    B = synth.dense_b(K, N, 902, kind="int")
    ref = oracle.spmm(A, B)[0]
    h = jig.reorder(_dev(A), 4)
    dB = _dev(B)
    with jig.launch_override(tile_n=64):
        C1 = torch.empty((M, N), dtype=torch.float16, device="cuda")
        h.spmm(dB, C=C1)
        d = jig.last_launch()
        assert d["dynamic_schedule"] == 1 and d["grid"] < d["work_items"], d
        outs = []
        for st in (torch.cuda.Stream(), torch.cuda.Stream()):
            with torch.cuda.stream(st):
                for _ in range(3):
                    c = torch.full((M, N), 5.0, dtype=torch.float16, device="cuda")
                    h.spmm(dB, C=c, stream=st)
                    outs.append(c)
        Cg = torch.empty((M, N), dtype=torch.float16, device="cuda")
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            h.spmm(dB, C=Cg)
        assert jig.last_launch()["graph_owned_workspace"] == 1
    for _ in range(3):
        Cg.fill_(3.0)
        g.replay()
        torch.cuda.synchronize()
        int_exact(_host(Cg), A, B)
    torch.cuda.synchronize()
    for c in [C1] + outs:
        assert np.array_equal(_host(c).view(np.float16).astype(np.float64), ref)


def test_many_streams_reclaim_regions():
    """Launches that need a workspace on 80 different streams (more than the 64
    per-stream regions kept per device): idle regions of earlier streams are
    reclaimed while later streams run; every result bit-exact."""
    mats, Bs, hs, refs = _int_batch(n_small=2, seed0=950)
    dB = [_dev(b) for b in Bs]
    outs = []
    with jig.launch_override(k_pieces=1):
        for i in range(80):
            st = torch.cuda.Stream()
            with torch.cuda.stream(st):
                dC = [torch.empty((a.shape[0], b.shape[1]), dtype=torch.float16, device="cuda")
                      for a, b in zip(mats, Bs)]
                jig.spmm_batched(hs, dB, dC, stream=st)
                assert jig.last_launch()["split_slots"] > 0
                outs.append((st, dC))
            if i % 16 == 15:
                torch.cuda.synchronize()
    torch.cuda.synchronize()
    for st, dC in outs:
        for r, c in zip(refs, dC):
            assert np.array_equal(_host(c).view(np.float16).astype(np.float64), r)
