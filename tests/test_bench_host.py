"""Host logic of bench.py: workloads match BASELINE.json's configs and the
multi-GPU job split covers every matrix / column exactly once (no GPU)."""
import numpy as np

import bench


def test_workloads():
    pts, desc, sc = bench.workload("c2")
    assert len(pts) == 36 and sc == "weak" and all(N == 256 for *_, N in pts)
    assert {(M, K) for (M, K, *_) in pts} == {(512, 2048), (2048, 512)}
    assert len(bench.workload("c3")[0]) == 19 * 2 * 4 * 2
    assert len(bench.workload("c4")[0]) == 8
    assert len(bench.workload("c5a")[0]) == 64 and bench.workload("c5a")[2] == "strong"
    assert bench.workload("c5b")[0] == [(4096, 4096, 8, 0.90, 16384)]


def test_strong_scaling_jobs_partition_the_work():
    for name in ("c5a", "c5b"):
        pts, _, _ = bench.workload(name)
        for world in (1, 2, 4, 8):
            jobs = [bench.local_jobs(name, pts, r, world) for r in range(world)]
            if name == "c5a":
                seeds = sorted(j[5] for js in jobs for j in js)
                assert seeds == sorted(bench.point_seed(i, 0) for i in range(64))
            else:
                cols = np.concatenate([np.arange(j[6], j[7]) for js in jobs for j in js])
                assert np.array_equal(cols, np.arange(16384))
                assert len({j[5] for js in jobs for j in js}) == 1     # same A on every rank


def test_weak_scaling_jobs_differ_by_rank():
    pts, _, _ = bench.workload("c2")
    a, b = bench.local_jobs("c2", pts, 0, 2), bench.local_jobs("c2", pts, 1, 2)
    assert len(a) == len(b) == 36 and {j[5] for j in a}.isdisjoint({j[5] for j in b})


def test_venom_workload_points_are_natively_24():
    """f4 workload: every point's A is V:2:Mb with 4 | Mb, so it is
    2:4 in natural column order (the cuSPARSELt baseline's input); s = 1 - 2/Mb."""
    import synth
    pts, desc, scaling = bench.workload("venom")
    assert len(pts) == len(synth.venom_points()) == 12 and scaling == "weak"
    for i, (M, K, v, s, N) in enumerate(pts):
        _, _, V, mb, _ = synth.venom_points()[i]
        assert mb % 4 == 0 and abs(s - (1 - 2 / mb)) < 1e-12
        assert bench.point_tag("venom", i, v, s) == f"V{V}_Mb{mb}"
    A = synth.venom(256, 480, 32, 20, 5)
    nz = (A & 0x7FFF) != 0
    assert nz.reshape(256, -1, 4).sum(axis=2).max() <= 2
    assert abs(nz.mean() - 2 / 20) < 1e-12


def test_algorithmic_bytes_and_flops():
    """Roofline numerator: per tile 16P values +
    2P metadata + 64 B gather list, the touched B rows once, C once; executed
    flops 2*P*16*N per tile; CUDA-core entries (f3) add 8 B each plus the per-row
    offsets and 2*N flops each."""
    info = dict(panel_rows=128, ntiles=10, npanels=2, cc_entries=0)
    ab, ef = bench.algorithmic(info, M=200, K=300, N=64, rows_touched=250)
    assert ab == (16 * 128 + 2 * 128 + 64) * 10 + 2 * 64 * 250 + 2 * 200 * 64
    assert ef == 2 * 128 * 16 * 10 * 64
    info["cc_entries"] = 7
    ab2, ef2 = bench.algorithmic(info, M=200, K=300, N=64, rows_touched=250)
    assert ab2 - ab == 8 * 7 + 4 * (2 * 128 + 1) and ef2 - ef == 2 * 7 * 64
    ab3, _ = bench.algorithmic(info, M=200, K=300, N=64, rows_touched=250, c_bytes_per_elem=4)
    assert ab3 - ab2 == 2 * 200 * 64


def test_paper_context_is_table2():
    """The paper's Table 2 cuBLAS column, quoted as context:
    twelve (v, s) cells, avg <= max, increasing with sparsity for every v."""
    t = bench.PAPER_TABLE2
    cells = {k: v for k, v in t.items() if k != "source"}
    assert len(cells) == 12 and "P:244-259" in t["source"]
    for v in (2, 4, 8):
        avgs = [cells[f"v{v}_s{s}"][0] for s in (80, 90, 95, 98)]
        assert avgs == sorted(avgs)
        assert all(a <= m for a, m in (cells[f"v{v}_s{s}"] for s in (80, 90, 95, 98)))
    assert cells["v8_s98"] == [2.14, 5.45] and cells["v2_s80"] == [0.77, 1.27]
