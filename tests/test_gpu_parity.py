"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

  * reorder / format: BIT-EXACT against oracle O2 (CR1) -- T_p, col_idx, perm,
    gather, vals, meta, kind, evictions -- and valid under checker O3;
  * SpMM: |C - C_ref| <= 1e-2 * (|A|.|B|) + 1e-3 element-wise (north_star
    tolerance), and bit-exact on integer-valued inputs.
Small cases span several tiles and a ragged tail; full-size cases (BASELINE
configs C2/C4) are checked on sampled panels and rows."""
import numpy as np
import pytest

import oracle
import synth
from oracle import check

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.set_device(0)


def _dev(x: np.ndarray):
    return torch.from_numpy(np.ascontiguousarray(x).view(np.int16)).cuda().view(torch.float16)


def _host(t) -> np.ndarray:
    if t.dtype == torch.float32:
        return t.cpu().numpy()
    return t.view(torch.int16).cpu().numpy().view(np.uint16)


@pytest.fixture
def override():
    """jigsaw_set_launch_override for one test (this thread), reset afterwards."""
    yield jig.set_launch_override
    jig.set_launch_override()


def assert_format_equal(gpu: dict, ref: oracle.Format, panels=None):
    if panels is None:
        assert np.array_equal(gpu["T"], ref.T)
        sl = slice(None)
    else:
        p0, p1 = panels
        toff = np.concatenate([[0], np.cumsum(gpu["T"])])
        assert np.array_equal(gpu["T"][p0:p1], ref.T)
        sl = slice(int(toff[p0]), int(toff[p1]))
    for k in ("col_idx", "perm", "vals", "meta", "kind", "nevict"):
        a, b = gpu[k][sl], getattr(ref, k)
        assert a.shape == b.shape, k
        bad = np.argwhere(a != b)
        assert bad.size == 0, f"{k} differs at {bad[:5].tolist()}"
    assert np.array_equal(gpu["gather"][sl], ref.gather)


def int_exact(C_gpu: np.ndarray, A, B, rows=None):
    """Integer-valued fixture (A in {+-1,+-2}, B in {-2..2}): every partial sum is
    an integer below 2^24, exact in fp32 in any order, so the GPU result must
    equal the oracle bit for bit.  fp16 C: the fixture must stay within
    |C| <= 2048 (integers exactly representable in fp16) -- asserted, not
    skipped; fp32 C (c_dtype = 1): exact as is."""
    C_ref, _ = oracle.spmm(A, B, rows=rows)
    C = C_gpu if rows is None else C_gpu[rows]
    if C.dtype == np.float32:
        got = C.astype(np.float64)
    else:
        assert np.abs(C_ref).max() <= 2048, "integer fixture leaves the exactly representable fp16 range"
        got = C.view(np.float16).astype(np.float64)
    bad = np.argwhere(got != C_ref)
    assert bad.size == 0, f"{len(bad)} mismatches, first at {bad[:3].tolist()}"


def spmm_check(C_gpu: np.ndarray, A, B, rows=None):
    C_ref, Mabs = oracle.spmm(A, B, rows=rows)
    C = C_gpu.astype(np.float64) if C_gpu.dtype == np.float32 else C_gpu.view(np.float16).astype(np.float64)
    if rows is not None:
        C = C[rows]
    err = np.abs(C - C_ref)
    tol = 1e-2 * Mabs + 1e-3
    worst = np.unravel_index(np.argmax(err - tol), err.shape)
    assert np.all(err <= tol), f"max excess at {worst}: err {err[worst]} tol {tol[worst]}"
    return float((err / (Mabs + 1e-30)).max())


CASES = [
    # M, K, v, s, N, kind, seed
    (256, 256, 4, 0.80, 64, "uniform", 1),     # C1
    (384, 512, 8, 0.90, 256, "uniform", 2),
    (200, 300, 4, 0.85, 136, "uniform", 3),    # ragged M, K % 16 != 0, N % 128 != 0
    (512, 1024, 2, 0.70, 128, "skewed", 4),
    (256, 512, 8, 0.50, 128, "uniform", 5),    # residual-heavy (many evictions)
    (128, 64, 1, 0.0, 64, "uniform", 6),       # fully dense panel
    (256, 2048, 8, 0.98, 256, "uniform", 7),
]


@pytest.mark.parametrize("M,K,v,s,N,kind,seed", CASES)
def test_reorder_bit_exact_and_spmm(M, K, v, s, N, kind, seed):
    A = synth.vector_sparse(M, K, v, s, seed, kind=kind)
    B = synth.dense_b(K, N, seed)
    h = jig.reorder(_dev(A), v)
    g = h.export()
    ref = oracle.reorder(A, P=128)
    assert_format_equal(g, ref)
    check.check_format(A, 128, g["T"], g["gather"], g["vals"], g["meta"], perm=g["perm"])
    info = h.info()
    assert info["ntiles"] == int(ref.T.sum())
    assert info["evictions"] == int(ref.nevict.sum())
    assert info["nnz"] == int(((A & 0x7FFF) != 0).sum())
    assert info["format_bytes"] == check.format_bytes(ref.T, 128)
    C = h.spmm(_dev(B))
    torch.cuda.synchronize()
    spmm_check(_host(C), A, B)
    h.free()


@pytest.mark.parametrize("M,K,V,Mb,N,P", [(512, 1000, 128, 20, 256, 128), (384, 600, 32, 12, 200, 128),
                                          (512, 2048, 64, 100, 256, 128), (512, 800, 256, 40, 256, 256)])
def test_venom_matrices(M, K, V, Mb, N, P):
    """VENOM-style V:2:Mb matrices.  GPU format
    bit-exact vs the oracle (identity reorder when P | V), C within tolerance,
    integer-valued inputs bit-exact."""
    A = synth.venom(M, K, V, Mb, 41)
    B = synth.dense_b(K, N, 41)
    h = jig.reorder(_dev(A), 1, panel_rows=P)
    g = h.export()
    ref = oracle.reorder(A, P=P)
    assert_format_equal(g, ref)
    if V % P == 0:
        assert h.info()["evictions"] == 0
    spmm_check(_host(h.spmm(_dev(B))), A, B)
    Ai = synth.venom(M, K, V, Mb, 42, kind="int")
    Bi = synth.dense_b(K, N, 42, kind="int")
    hi = jig.reorder(_dev(Ai), 1, panel_rows=P)
    Ci = _host(hi.spmm(_dev(Bi)))
    torch.cuda.synchronize()
    int_exact(Ci, Ai, Bi)


@pytest.mark.parametrize("seed", [11, 12])
def test_spmm_integer_inputs_bit_exact(seed):
    """Integer-valued A in {+-1,+-2}, B in {-2..2}, |C| <= 2048: every fp32 partial
    sum is exact, so the GPU result must equal the oracle bit for bit."""
    M, K, N = 384, 640, 192
    A = synth.vector_sparse(M, K, 4, 0.9, seed, kind="int")
    B = synth.dense_b(K, N, seed, kind="int")
    h = jig.reorder(_dev(A), 4)
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    C_ref, _ = oracle.spmm(A, B)
    assert np.abs(C_ref).max() <= 2048
    assert np.array_equal(C.view(np.float16).astype(np.float64), C_ref)


def test_all_zero_panel_and_empty_matrix():
    A = np.zeros((384, 96), np.uint16)
    A[130:138, 5] = np.float16(1.0).view(np.uint16)   # only panel 1 has nonzeros
    B = synth.dense_b(96, 64, 1)
    h = jig.reorder(_dev(A), 8)
    g = h.export()
    assert g["T"].tolist() == [0, 1, 0]
    Cd = torch.full((384, 64), 7.0, dtype=torch.float16, device="cuda")
    h.spmm(_dev(B), C=Cd)
    C = _host(Cd)
    spmm_check(C, A, B)
    assert np.all(C[:128] == 0) and np.all(C[256:] == 0)
    Z = np.zeros((128, 64), np.uint16)
    hz = jig.reorder(_dev(Z), 1)
    assert hz.info()["ntiles"] == 0
    Cz = hz.spmm(_dev(synth.dense_b(64, 32, 2)))
    assert int(torch.count_nonzero(Cz)) == 0


def test_already_24_and_v_independence():
    A = synth.nm24(256, 256, 3)
    h = jig.reorder(_dev(A), 1)
    g = h.export()
    assert int(g["nevict"].sum()) == 0
    assert all(g["perm"][t].tolist() == list(range(16)) for t in range(len(g["perm"])))
    A8 = synth.vector_sparse(256, 256, 8, 0.9, 9)
    g1, g8 = jig.reorder(_dev(A8), 1).export(), jig.reorder(_dev(A8), 8).export()
    for k in g1:
        assert np.array_equal(g1[k], g8[k]), k     # R-Q22: the format ignores v


def test_negative_zero_and_host_paths():
    A = synth.vector_sparse(256, 128, 4, 0.8, 5)
    A[3, :] = np.where(A[3, :] == 0, np.uint16(0x8000), A[3, :])   # -0 entries are zeros
    B = synth.dense_b(128, 64, 5)
    h = jig.reorder_host(A, 4)
    assert_format_equal(h.export(), oracle.reorder(A, P=128))
    C = h.spmm_host(B)
    spmm_check(C, A, B)


def test_spmm_batched_and_streams():
    mats = [synth.vector_sparse(256, 384, 8, 0.9, 20 + i) for i in range(3)]
    Bs = [synth.dense_b(384, 128, 30 + i) for i in range(3)]
    hs = [jig.reorder(_dev(a), 8) for a in mats]
    dB = [_dev(b) for b in Bs]
    dC = [torch.empty((256, 128), dtype=torch.float16, device="cuda") for _ in range(3)]
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        jig.spmm_batched(hs, dB, dC, stream=s)
    s.synchronize()
    for a, b, c in zip(mats, Bs, dC):
        spmm_check(_host(c), a, b)


@pytest.mark.parametrize("M1,K,N,P", [(512, 2048, 256, 128), (2048, 512, 256, 128), (1024, 1536, 512, 256)])
def test_programmatic_dependent_launch_ordering(M1, K, N, P):
    """k_spmm is launched with the programmatic-dependent-launch attribute: its
    prologue (handle-owned A / metadata / gather lists) overlaps the previous
    kernel, every access to B and C waits on griddepcontrol.wait.  Checked with no
    host sync anywhere: B written by the kernel right before the call (behind a
    long matmul), C read by the kernel right before (write-after-read: the clone
    must see the old contents), C consumed right after, and a chain where the
    output of one SpMM is the B of the next (single split-K, grouped and pair
    launches)."""
    v = 8
    A1 = synth.vector_sparse(M1, K, v, 0.9, 61)
    A2 = synth.vector_sparse(384, M1, v, 0.9, 62)
    Bh = synth.dense_b(K, N, 63)
    h1 = jig.reorder(_dev(A1), v, panel_rows=P)
    h2 = jig.reorder(_dev(A2), v)
    src = _dev(Bh)
    B = torch.zeros_like(src)
    C1 = torch.full((M1, N), 7.0, dtype=torch.float16, device="cuda")
    C2 = torch.empty((384, N), dtype=torch.float16, device="cuda")
    big = torch.randn(4096, 4096, device="cuda", dtype=torch.float16)
    torch.cuda.synchronize()
    _ = big @ big                 # keeps the stream busy so the copy below is still pending
    B.copy_(src)                  # producer of B, immediately before the SpMM
    old = C1.clone()              # reader of C, immediately before the SpMM
    h1.spmm(B, C=C1)
    h2.spmm(C1, C=C2)             # consumer of C1 as the next B
    torch.cuda.synchronize()
    assert bool((old == 7.0).all())
    C1h = _host(C1)
    spmm_check(C1h, A1, Bh)
    spmm_check(_host(C2), A2, C1h)


def test_abi_errors_on_gpu():
    A = synth.vector_sparse(128, 64, 4, 0.8, 1)
    h = jig.reorder(_dev(A), 4)
    B = _dev(synth.dense_b(64, 64, 1))
    with pytest.raises(jig.JigsawError) as e:
        h.spmm(B[:, :60].contiguous())      # N % 8 != 0
    assert e.value.status == 1
    L = jig.lib()
    Cd = torch.empty((128, 64), dtype=torch.float16, device="cuda")
    import ctypes
    st = L.jigsaw_spmm(h.ptr, ctypes.c_void_p(B.data_ptr() + 2), 64, ctypes.c_void_p(Cd.data_ptr()), None)
    assert st == 1                            # misaligned B
    with pytest.raises(jig.JigsawError):
        jig.reorder(_dev(synth.vector_sparse(8, 8, 1, 0.5, 1)), 3)
    h64 = jig.reorder(_dev(A), 4, panel_rows=64)   # analysis-only format: no M = 64 MMA
    with pytest.raises(jig.JigsawError) as e:
        h64.spmm(B)
    assert e.value.status == 2
    with pytest.raises(jig.JigsawError) as e:
        jig.reorder(_dev(A), 4, panel_rows=100)
    assert e.value.status == 1


# ---------------------------------------------------------------- full sizes
@pytest.mark.parametrize("M,K,v,s,N", [
    (2048, 512, 8, 0.95, 256),      # C2
    (512, 2048, 2, 0.80, 256),      # C2
    (4096, 4096, 8, 0.90, 2048),    # C4
    (11008, 4096, 8, 0.70, 2048),   # C4
])
def test_full_size_sampled(M, K, v, s, N):
    """BASELINE sizes in the launch configuration bench.py times: format
    bit-exact on two sampled panels, C checked on 24 sampled rows."""
    A = synth.vector_sparse(M, K, v, s, 1)
    B = synth.dense_b(K, N, 1)
    h = jig.reorder(_dev(A), v)
    g = h.export()
    npan = (M + 127) // 128
    for p in sorted({0, npan // 2, npan - 1}):
        ref = oracle.reorder(A, P=128, panels=(p, p + 1))
        assert_format_equal(g, ref, panels=(p, p + 1))
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    rng = np.random.default_rng(0)
    rows = np.sort(rng.choice(M, size=24, replace=False))
    spmm_check(C, A, B, rows=rows)


@pytest.mark.parametrize("M,P", [(2049 * 128 - 40, 128), (1040 * 256 + 8, 256)])
def test_parameter_table_capacity_fallbacks(M, P):
    """Tall matrices past the grouped launch's parameter tables: more panels than
    the in-parameter panel table holds (1024: the kernel reads the device copy)
    and, at P = 128, more work units than the host schedule list holds (2048:
    units are decoded by scanning the problem table).  Format bit-exact on
    sampled panels, C on sampled rows (incl. the ragged last panel)."""
    K, v, s, N = 64, 8, 0.9, 64
    A = synth.vector_sparse(M, K, v, s, 17)
    B = synth.dense_b(K, N, 17)
    h = jig.reorder(_dev(A), v, panel_rows=P)
    g = h.export()
    npan = (M + P - 1) // P
    for p in sorted({0, 1500 % npan, npan - 1}):
        ref = oracle.reorder(A, P=P, panels=(p, p + 1))
        assert_format_equal(g, ref, panels=(p, p + 1))
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    rng = np.random.default_rng(1)
    rows = np.sort(np.concatenate([rng.choice(M, size=40, replace=False), np.arange(M - 8, M)]))
    spmm_check(C, A, B, rows=rows)


@pytest.mark.parametrize("force", [1, 2, 4, 8])
@pytest.mark.parametrize("M,K,v,s,N", [(512, 2048, 4, 0.9, 256), (384, 700, 8, 0.8, 200),
                                       (256, 96, 2, 0.95, 64)])
def test_spmm_kernel_variants(force, M, K, v, s, N, override):
    """Every k_spmm variant (NT = 64 with split-K S = 1/2/4/8 over a cluster and the
    DSMEM reduce-scatter) against the oracle, incl. splits that get no k-block."""
    override(split_k=force)
    A = synth.vector_sparse(M, K, v, s, 3)
    B = synth.dense_b(K, N, 3)
    h = jig.reorder(_dev(A), v)
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    assert jig.last_launch()["split_k"] == force
    spmm_check(C, A, B)
    Ai = synth.vector_sparse(M, K, v, s, 4, kind="int")
    Bi = synth.dense_b(K, N, 4, kind="int")
    hi = jig.reorder(_dev(Ai), v)
    Ci = _host(hi.spmm(_dev(Bi)))
    torch.cuda.synchronize()
    int_exact(Ci, Ai, Bi)


@pytest.mark.parametrize("force", [1, 2, 4])
@pytest.mark.parametrize("M,K,v,s,N", [(512, 2048, 4, 0.9, 256), (384, 700, 8, 0.8, 200),
                                       (256, 96, 2, 0.95, 40), (2048, 512, 8, 0.7, 104)])
def test_spmm_nt32_variants(force, M, K, v, s, N, override):
    """32-column tiles (the latency path of small single products; B staged in
    half of a 64-column SW128 chunk, N = 32 MMAs) with split-K S = 1/2/4, ragged
    N tails (N % 32 != 0), single and grouped launches, against the oracle;
    integer-valued inputs bit-exact."""
    override(tile_n=32, split_k=force)
    A = synth.vector_sparse(M, K, v, s, 13)
    B = synth.dense_b(K, N, 13)
    h = jig.reorder(_dev(A), v)
    spmm_check(_host(h.spmm(_dev(B))), A, B)
    Ai = synth.vector_sparse(M, K, v, s, 14, kind="int")
    Bi = synth.dense_b(K, N, 14, kind="int")
    hi = jig.reorder(_dev(Ai), v)
    Ci = _host(hi.spmm(_dev(Bi)))
    torch.cuda.synchronize()
    int_exact(Ci, Ai, Bi)
    override(tile_n=32)
    dC = [torch.empty((M, N), dtype=torch.float16, device="cuda") for _ in range(2)]
    jig.spmm_batched([h, hi], [_dev(B), _dev(Bi)], dC)
    torch.cuda.synchronize()
    spmm_check(_host(dC[0]), A, B)
    spmm_check(_host(dC[1]), Ai, Bi)


def test_grouped_launch_many_mixed_problems():
    """jigsaw_spmm_batched: one grouped persistent launch per 64 products; 70 mixed
    shapes / N / sparsities (incl. an all-zero matrix) against the oracle."""
    rng = np.random.default_rng(5)
    shapes = [(128, 64), (256, 96), (200, 160), (384, 128), (64, 256)]
    mats, Bs, hs = [], [], []
    for i in range(70):
        M, K = shapes[i % len(shapes)]
        v = [1, 2, 4, 8][i % 4]
        M -= M % v
        s = float(rng.choice([0.5, 0.8, 0.95]))
        A = synth.vector_sparse(M, K, v, s, 100 + i) if i != 7 else np.zeros((M, K), np.uint16)
        N = int(rng.choice([64, 136, 256]))
        mats.append(A)
        Bs.append(synth.dense_b(K, N, 200 + i))
        hs.append(jig.reorder(_dev(A), v))
    dB = [_dev(b) for b in Bs]
    dC = [torch.full((a.shape[0], b.shape[1]), 3.0, dtype=torch.float16, device="cuda")
          for a, b in zip(mats, Bs)]
    jig.spmm_batched(hs, dB, dC)
    torch.cuda.synchronize()
    for a, b, c in zip(mats, Bs, dC):
        spmm_check(_host(c), a, b)


@pytest.mark.parametrize("M,K,v,s,N,seed", [
    (256, 512, 8, 0.50, 128, 1),     # residual-heavy: many dense tiles
    (384, 300, 4, 0.70, 136, 2),     # ragged K / N
    (256, 256, 4, 0.90, 64, 3),      # few or no residual tiles
    (512, 2048, 2, 0.50, 256, 4),    # C2 shape, v = 2, 50 %
])
def test_dense_residual_mode(M, K, v, s, N, seed):
    """DENSE residual mode: evicted columns go to uncompressed 16-column
    tiles run on the dense tensor path.  Format bit-exact vs oracle mode 1 (incl.
    the residual columns and values), C within tolerance, integers bit-exact."""
    A = synth.vector_sparse(M, K, v, s, seed)
    B = synth.dense_b(K, N, seed)
    h = jig.reorder(_dev(A), v, residual_mode=1)
    g = h.export()
    ref = oracle.reorder(A, P=128, mode=1)
    assert_format_equal(g, ref)
    assert np.array_equal(g["D"], ref.D)
    assert np.array_equal(g["rcol"], ref.rcol)
    assert np.array_equal(g["dvals"], ref.dvals)
    check.check_format(A, 128, g["T"], g["gather"], g["vals"], g["meta"], perm=g["perm"],
                       D=g["D"], rcol=g["rcol"], dvals=g["dvals"])
    assert h.info()["ndtiles"] == int(ref.D.sum())
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    spmm_check(C, A, B)
    Ai = synth.vector_sparse(M, K, v, s, seed + 50, kind="int")
    Bi = synth.dense_b(K, N, seed + 50, kind="int")
    hi = jig.reorder(_dev(Ai), v, residual_mode=1)
    Ci = _host(hi.spmm(_dev(Bi)))
    torch.cuda.synchronize()
    int_exact(Ci, Ai, Bi)


@pytest.mark.parametrize("force", [2, 4])
def test_dense_residual_split_and_grouped(force, override):
    """DENSE-mode k-blocks under split-K clusters and in a grouped launch."""
    mats = [synth.vector_sparse(256, 640, 4, 0.6, 70 + i) for i in range(3)]
    Bs = [synth.dense_b(640, 128, 80 + i) for i in range(3)]
    hs = [jig.reorder(_dev(a), 4, residual_mode=1) for a in mats]
    override(split_k=force)
    for h, a, b in zip(hs, mats, Bs):
        spmm_check(_host(h.spmm(_dev(b))), a, b)
    override()
    dB = [_dev(b) for b in Bs]
    dC = [torch.empty((256, 128), dtype=torch.float16, device="cuda") for _ in range(3)]
    jig.spmm_batched(hs, dB, dC)
    torch.cuda.synchronize()
    for a, b, c in zip(mats, Bs, dC):
        spmm_check(_host(c), a, b)


@pytest.mark.parametrize("nt", [64, 128, 256])
def test_tile_width_variants(nt, override):
    """k_spmm with N tiles of 64 / 128 / 256 columns (single and grouped launches,
    SPTC and DENSE residual), N not a multiple of the tile width."""
    override(tile_n=nt)
    mats = [synth.vector_sparse(384, 700, 8, 0.85, 90 + i) for i in range(2)]
    Bs = [synth.dense_b(700, 328, 91 + i) for i in range(2)]
    hs = [jig.reorder(_dev(mats[0]), 8), jig.reorder(_dev(mats[1]), 8, residual_mode=1)]
    for h, a, b in zip(hs, mats, Bs):
        spmm_check(_host(h.spmm(_dev(b))), a, b)
    dB = [_dev(b) for b in Bs]
    dC = [torch.empty((384, 328), dtype=torch.float16, device="cuda") for _ in range(2)]
    jig.spmm_batched(hs, dB, dC)
    torch.cuda.synchronize()
    for a, b, c in zip(mats, Bs, dC):
        spmm_check(_host(c), a, b)


# ---------------------------------------------------------------- 256-row panels
PAIR_CASES = [
    # M, K, v, s, N, kind, seed, mode
    (512, 384, 8, 0.90, 256, "uniform", 21, 0),
    (600, 300, 4, 0.80, 136, "uniform", 22, 0),     # ragged M (last panel 88 rows), ragged K / N
    (256, 512, 8, 0.50, 128, "uniform", 23, 0),     # residual-heavy
    (1024, 2048, 2, 0.70, 512, "skewed", 24, 0),
    (600, 256, 4, 0.80, 200, "uniform", 25, 1),     # DENSE residual mode
    (130, 64, 2, 0.0, 64, "uniform", 26, 0),        # one dense panel with 2 rows in its 2nd half
]


@pytest.mark.parametrize("M,K,v,s,N,kind,seed,mode", PAIR_CASES)
@pytest.mark.parametrize("nt", [128, 256])
def test_pair_panels_bit_exact_and_spmm(M, K, v, s, N, kind, seed, mode, nt, override):
    """panel_rows = 256 (R-Q6): one CTA pair per panel (tcgen05 cta_group::2, M = 256).
    Format bit-exact vs oracle O2 at P = 256 (incl. the two per-half planes the
    kernel reads), C within tolerance for N tiles of 128 and 256, integers bit-exact."""
    override(tile_n=nt)
    A = synth.vector_sparse(M, K, v, s, seed, kind=kind)
    B = synth.dense_b(K, N, seed)
    h = jig.reorder(_dev(A), v, panel_rows=256, residual_mode=mode)
    g = h.export()
    ref = oracle.reorder(A, P=256, mode=mode)
    assert_format_equal(g, ref)
    if mode == 1:
        assert np.array_equal(g["D"], ref.D)
        assert np.array_equal(g["rcol"], ref.rcol)
        assert np.array_equal(g["dvals"], ref.dvals)
    check.check_format(A, 256, g["T"], g["gather"], g["vals"], g["meta"], perm=g["perm"],
                       D=g["D"] if mode == 1 else None, rcol=g["rcol"] if mode == 1 else None,
                       dvals=g["dvals"] if mode == 1 else None)
    info = h.info()
    assert info["panel_rows"] == 256
    assert info["format_bytes"] == check.format_bytes(ref.T, 256, ref.D if mode == 1 else None)
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    spmm_check(C, A, B)
    h.free()
    Ai = synth.vector_sparse(M, K, v, s, seed + 50, kind="int")
    Bi = synth.dense_b(K, N, seed + 50, kind="int")
    hi = jig.reorder(_dev(Ai), v, panel_rows=256, residual_mode=mode)
    Ci = _host(hi.spmm(_dev(Bi)))
    torch.cuda.synchronize()
    assert jig.last_launch()["cta_pair"] == 1 and jig.last_launch()["tile_n"] == nt
    int_exact(Ci, Ai, Bi)


def test_pair_panels_grouped_mixed_with_single():
    """A batch mixing 128-row and 256-row panel formats (two grouped launches),
    including an all-zero matrix, against the oracle."""
    mats, Bs, hs = [], [], []
    for i in range(12):
        M, K = [(512, 300), (256, 640), (384, 128)][i % 3]
        v = [2, 4, 8][i % 3]
        A = synth.vector_sparse(M, K, v, 0.85, 300 + i) if i != 5 else np.zeros((M, K), np.uint16)
        mats.append(A)
        Bs.append(synth.dense_b(K, 192, 400 + i))
        hs.append(jig.reorder(_dev(A), v, panel_rows=256 if i % 2 else 128))
    dB = [_dev(b) for b in Bs]
    dC = [torch.full((a.shape[0], 192), 3.0, dtype=torch.float16, device="cuda") for a in mats]
    jig.spmm_batched(hs, dB, dC)
    torch.cuda.synchronize()
    for a, b, c in zip(mats, Bs, dC):
        spmm_check(_host(c), a, b)


def test_pair_panels_full_size_sampled():
    """BASELINE C4-sized product with 256-row panels, sampled rows of both halves."""
    M, K, N, v, s = 4096, 4096, 4096, 8, 0.9
    A = synth.vector_sparse(M, K, v, s, 31)
    B = synth.dense_b(K, N, 31)
    h = jig.reorder(_dev(A), v, panel_rows=0)           # auto: M >= 4096 -> 256-row panels
    assert h.info()["panel_rows"] == 256
    assert jig.reorder(_dev(A[:512]), v, panel_rows=0).info()["panel_rows"] == 128
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    rows = np.array([0, 127, 128, 255, 256 * 7 + 5, 256 * 7 + 200, M - 129, M - 1])
    spmm_check(C, A, B, rows=rows)
    ref = oracle.reorder(A, P=256, panels=(7, 8))
    assert_format_equal(h.export(), ref, panels=(7, 8))


@pytest.mark.parametrize("P", [128, 256])
@pytest.mark.parametrize("pieces", ["nsplit", "kpieces", "off"])
def test_grouped_split_pieces(P, pieces, override):
    """Grouped launch where a few long units dominate: they are cut into column
    slices (N-split, the default: each slice re-reads the unit's A over the whole
    k-range, no workspace) or, with the k_pieces override, into k-range pieces
    whose fp32 partial tiles are reduced through the workspace (last-arriver);
    with splitting disabled (no_pieces) the same batch runs whole units.  All
    against the oracle, integers bit-exact; replayed twice (the per-unit
    counters reset)."""
    if pieces == "off":
        override(no_pieces=1)
    elif pieces == "kpieces":
        override(k_pieces=1)
    mats, Bs = [], []
    mats.append(synth.vector_sparse(512, 6000, 2, 0.5, 501, kind="int"))   # ~90 k-blocks per panel
    Bs.append(synth.dense_b(6000, 200, 502, kind="int"))
    mats.append(synth.vector_sparse(300, 3000, 4, 0.6, 503))
    Bs.append(synth.dense_b(3000, 136, 504))
    for i in range(20):
        mats.append(synth.vector_sparse(128, 96, 4, 0.8, 510 + i))
        Bs.append(synth.dense_b(96, 64, 530 + i))
    hs = [jig.reorder(_dev(a), 2 if i == 0 else 4, panel_rows=P) for i, a in enumerate(mats)]
    dB = [_dev(b) for b in Bs]
    for rep in range(2):
        dC = [torch.full((a.shape[0], b.shape[1]), 7.0, dtype=torch.float16, device="cuda")
              for a, b in zip(mats, Bs)]
        jig.spmm_batched(hs, dB, dC)
        torch.cuda.synchronize()
        d = jig.last_launch()
        assert (d["split_slots"] > 0) == (pieces == "kpieces"), d
        assert (d["nsplit_items"] > 0) == (pieces == "nsplit"), d
        for i, (a, b, c) in enumerate(zip(mats, Bs, dC)):
            if i == 0:
                int_exact(_host(c), a, b)
            else:
                spmm_check(_host(c), a, b)


@pytest.mark.parametrize("P", [16, 32, 64])
@pytest.mark.parametrize("M,K,v,s,mode", [(256, 512, 8, 0.90, 0), (200, 300, 4, 0.70, 0), (128, 256, 2, 0.5, 1)])
def test_small_panel_formats_bit_exact(P, M, K, v, s, mode):
    """The paper's BLOCK_TILE heights through the GPU builder: format
    bit-exact vs oracle O2 at the same P (the reorder-study path)."""
    A = synth.vector_sparse(M, K, v, s, 40 + P)
    h = jig.reorder(_dev(A), v, panel_rows=P, residual_mode=mode)
    g = h.export()
    ref = oracle.reorder(A, P=P, mode=mode)
    assert_format_equal(g, ref)
    if mode == 1:
        assert np.array_equal(g["rcol"], ref.rcol)
        assert np.array_equal(g["dvals"], ref.dvals)
    check.check_format(A, P, g["T"], g["gather"], g["vals"], g["meta"], perm=g["perm"],
                       D=g["D"] if mode == 1 else None, rcol=g["rcol"] if mode == 1 else None,
                       dvals=g["dvals"] if mode == 1 else None)
    h.free()


def test_spmm_batched_host_pipeline():
    """jigsaw_spmm_batched_host: host B's in, host C's out, chunks of the batch
    pipelined over three streams -- every C against the oracle, mixed panel
    heights (single and pair launches), ragged N, pinned and pageable buffers."""
    pts = [(512, 2048, 4, 0.9, 256), (2048, 512, 8, 0.8, 200), (384, 700, 8, 0.8, 72), (1024, 1024, 8, 0.9, 512)]
    mats = [synth.vector_sparse(M, K, v, s, 70 + i) for i, (M, K, v, s, N) in enumerate(pts)]
    Bs = [synth.dense_b(K, N, 80 + i) for i, (M, K, v, s, N) in enumerate(pts)]
    hs = [jig.reorder(_dev(a), v, panel_rows=(256 if i == 3 else 128)) for i, (a, (M, K, v, s, N)) in
          enumerate(zip(mats, pts))]
    Cs = jig.spmm_batched_host(hs, Bs)                        # pageable
    for a, b, c in zip(mats, Bs, Cs):
        spmm_check(c, a, b)
    pin_B = [torch.from_numpy(b.view(np.int16)).pin_memory().numpy().view(np.uint16) for b in Bs]
    pin_C = [torch.empty((M, N), dtype=torch.int16).pin_memory().numpy().view(np.uint16) for (M, K, v, s, N) in pts]
    jig.spmm_batched_host(hs, pin_B, pin_C)                   # pinned, overlapped
    for a, b, c in zip(mats, Bs, pin_C):
        spmm_check(c, a, b)


@pytest.mark.parametrize("chunks", [1, 8])
def test_spmm_batched_host_packed_buffers(override, chunks):
    """jigsaw_spmm_batched_host with every B in one pinned block and every C in
    another (views into one registration, back to back; one product with a
    size that is not a multiple of 256 B), whole batch as one chunk and as
    several."""
    pts = [(256, 512, 4, 0.8, 128), (512, 256, 8, 0.9, 64), (384, 520, 8, 0.8, 72), (256, 256, 4, 0.7, 128)]
    mats = [synth.vector_sparse(M, K, v, s, 90 + i) for i, (M, K, v, s, N) in enumerate(pts)]
    Bs = [synth.dense_b(K, N, 95 + i) for i, (M, K, v, s, N) in enumerate(pts)]
    hs = [jig.reorder(_dev(a), v) for a, (M, K, v, s, N) in zip(mats, pts)]
    nb = sum(K * N for (M, K, v, s, N) in pts)
    nc = sum(M * N for (M, K, v, s, N) in pts)
    blkB = torch.empty(nb, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
    blkC = torch.empty(nc, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
    vb, vc, ob, oc = [], [], 0, 0
    for b, (M, K, v, s, N) in zip(Bs, pts):
        vb.append(blkB[ob:ob + K * N].reshape(K, N))
        vb[-1][...] = b.view(np.uint16) if b.dtype == np.float16 else b
        vc.append(blkC[oc:oc + M * N].reshape(M, N))
        ob += K * N
        oc += M * N
    blkC[...] = 0xFFFF
    override(host_chunks=chunks)                           # 1: the whole batch is one chunk
    jig.spmm_batched_host(hs, vb, vc)
    for a, b, c in zip(mats, Bs, vc):
        spmm_check(c, a, b)


def test_grouped_split_pieces_two_streams():
    """Grouped launches with k-range pieces (fp32 workspace, last-arriver
    reduction) queued on two streams that run at the same time: 5 launches on
    one stream, then 5 on the other, each into its own outputs.  Every stream
    has its own workspace regions, so no launch sees another's partials;
    integer inputs bit-exact against the oracle."""
    mats = [synth.vector_sparse(512, 6000, 2, 0.5, 601, kind="int")]
    Bs = [synth.dense_b(6000, 200, 602, kind="int")]
    for i in range(12):
        mats.append(synth.vector_sparse(128, 96, 4, 0.8, 610 + i, kind="int"))
        Bs.append(synth.dense_b(96, 64, 630 + i, kind="int"))
    hs = [jig.reorder(_dev(a), 2 if i == 0 else 4) for i, a in enumerate(mats)]
    dB = [_dev(b) for b in Bs]
    refs = [oracle.spmm(a, b)[0] for a, b in zip(mats, Bs)]
    assert max(np.abs(r).max() for r in refs) <= 2048, "integer fixture must stay exact in fp16"
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    big = torch.randn(4096, 4096, device="cuda", dtype=torch.float16)
    torch.cuda.synchronize()
    outs = []
    for st in streams:
        with torch.cuda.stream(st):
            _ = big @ big                      # both streams start behind a long matmul
    for st in streams:
        with torch.cuda.stream(st):           # the fills below are ordered on st too
            for _ in range(5):
                dC = [torch.full((a.shape[0], b.shape[1]), 7.0, dtype=torch.float16, device="cuda")
                      for a, b in zip(mats, Bs)]
                jig.spmm_batched(hs, dB, dC, stream=st)
                outs.append(dC)
    torch.cuda.synchronize()
    for dC in outs:
        for r, c in zip(refs, dC):
            assert np.array_equal(_host(c).view(np.float16).astype(np.float64), r)


def test_host_threads_concurrent_calls():
    """Four host threads call jigsaw_spmm_batched_host and jigsaw_spmm_batched at
    once (ctypes releases the GIL, so the calls really overlap in the library:
    lazily created pools, pipeline streams and workspace assignment under
    contention); every C against the oracle."""
    import threading
    pts = [(256, 512, 4, 0.8, 64), (384, 700, 8, 0.9, 72)]
    mats = [synth.vector_sparse(M, K, v, s, 700 + i) for i, (M, K, v, s, N) in enumerate(pts)]
    Bs = [synth.dense_b(K, N, 710 + i) for i, (M, K, v, s, N) in enumerate(pts)]
    hs = [jig.reorder(_dev(a), v) for a, (M, K, v, s, N) in zip(mats, pts)]
    dB = [_dev(b) for b in Bs]
    torch.cuda.synchronize()
    results, errors = {}, []

    def work(t):
        try:
            torch.cuda.set_device(0)
            if t % 2:
                results[t] = jig.spmm_batched_host(hs, Bs)
            else:
                st = torch.cuda.Stream()
                dC = [torch.empty((M, N), dtype=torch.float16, device="cuda") for (M, K, v, s, N) in pts]
                jig.spmm_batched(hs, dB, dC, stream=st)
                st.synchronize()
                results[t] = [_host(c) for c in dC]
        except Exception as e:                  # noqa: BLE001 -- reported below
            errors.append(repr(e))

    ths = [threading.Thread(target=work, args=(t,)) for t in range(4)]
    for th in ths:
        th.start()
    for th in ths:
        th.join()
    assert not errors, errors
    for t in range(4):
        for a, b, c in zip(mats, Bs, results[t]):
            spmm_check(c, a, b)


# ---------------------------------------------------------------- row-clustered panels (f2)
@pytest.mark.parametrize("M,K,v,s,kind,P,mode,ov", [
    (512, 2048, 4, 0.9, "skewed", 128, 0, {}),                 # grouped path (C2 shape)
    (2048, 512, 8, 0.8, "skewed", 128, 0, {}),
    (600, 300, 4, 0.85, "skewed", 128, 0, dict(split_k=2)),      # split-K cluster, ragged M/K
    (520, 256, 8, 0.9, "uniform", 256, 0, {}),                   # CTA pairs, ragged last pair panel
    (384, 640, 4, 0.6, "skewed", 128, 1, {}),                    # DENSE residual mode
    (256, 200, 2, 0.9, "skewed", 128, 0, dict(tile_n=32, split_k=1)),
])
def test_row_clustered_panels(M, K, v, s, kind, P, mode, ov, override):
    """jigsaw_options_t.row_order = JIGSAW_ROWS_CLUSTERED: the GPU
    row order equals oracle.row_cluster, the format is bit-exact vs CR1 of A[order],
    and C -- scattered back to A's row order by the epilogue -- matches the oracle
    product of the UNPERMUTED A (fp16 and fp32 C; integers bit-exact)."""
    A = synth.vector_sparse(M, K, v, s, 77, kind=kind)
    A[3] = 0                                                    # an all-zero row sorts last
    B = synth.dense_b(K, 136, 77)
    override(**ov)
    h = jig.reorder(_dev(A), v, panel_rows=P, residual_mode=mode, row_order=jig.ROWS_CLUSTERED)
    assert h.info()["row_order"] == jig.ROWS_CLUSTERED
    g = h.export()
    ref = oracle.reorder(A, P=P, mode=mode, row_order=1)
    assert np.array_equal(g["rowmap"], ref.rowmap)
    assert_format_equal(g, ref)
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    spmm_check(C, A, B)
    Ai = synth.vector_sparse(M, K, v, s, 78, kind="int")
    Bi = synth.dense_b(K, 136, 78, kind="int")
    hi = jig.reorder(_dev(Ai), v, panel_rows=P, residual_mode=mode, row_order=jig.ROWS_CLUSTERED,
                     c_dtype=jig.C_F32)
    Ci = _host(hi.spmm(_dev(Bi)))
    torch.cuda.synchronize()
    int_exact(Ci, Ai, Bi)
    h0 = jig.reorder(_dev(A), v, panel_rows=P, residual_mode=mode)
    assert np.array_equal(h0.export()["rowmap"], np.arange(M))     # identity for the given order



@pytest.mark.parametrize("M,K,v,s,N", [(512, 2048, 4, 0.9, 256), (4096, 2048, 8, 0.9, 1024)])
def test_panel_height_autotune(M, K, v, s, N):
    """panel_rows = JIGSAW_PANEL_AUTOTUNE (per-shape panel height):
    both formats are built and timed on the device, the faster kept; whichever it
    is, the format is bit-exact vs the oracle at that height and C correct."""
    A = synth.vector_sparse(M, K, v, s, 66)
    B = synth.dense_b(K, N, 66)
    h = jig.reorder(_dev(A), v, panel_rows=jig.PANEL_AUTOTUNE, autotune_n=N)
    P = h.info()["panel_rows"]
    assert P in (128, 256)
    npan = (M + P - 1) // P
    for p in sorted({0, npan - 1}):
        assert_format_equal(h.export(), oracle.reorder(A, P=P, panels=(p, p + 1)), panels=(p, p + 1))
    C = _host(h.spmm(_dev(B)))
    torch.cuda.synchronize()
    spmm_check(C, A, B, rows=np.unique(np.r_[np.arange(0, M, 37), M - 1]))


def test_reorder_batched_matches_single_builds():
    """jigsaw_reorder_batched (concurrent builds on internal streams) gives the
    same formats as one jigsaw_reorder_ex per matrix; an invalid matrix in the
    batch fails the call and leaves no handle."""
    pts = [(512, 2048, 4, 0.7), (2048, 512, 8, 0.9), (384, 300, 2, 0.5), (256, 256, 8, 0.98)] * 3
    mats = [synth.vector_sparse(M, K, v, s, 120 + i) for i, (M, K, v, s) in enumerate(pts)]
    dA = [_dev(a) for a in mats]
    hs = jig.reorder_batched(dA, [v for (M, K, v, s) in pts], row_order=jig.ROWS_CLUSTERED)
    for h, a, (M, K, v, s) in zip(hs, dA, pts):
        g1 = h.export()
        g2 = jig.reorder(a, v, row_order=jig.ROWS_CLUSTERED).export()
        for k in g1:
            assert np.array_equal(g1[k], g2[k]), k
    ref = oracle.reorder(mats[0], P=128, row_order=1)
    assert_format_equal(hs[0].export(), ref)
    bad = _dev(synth.vector_sparse(12, 64, 4, 0.5, 1))
    with pytest.raises(jig.JigsawError) as e:
        jig.reorder_batched([dA[1], bad], [8, 8])          # 12 % 8 != 0
    assert e.value.status == 1
