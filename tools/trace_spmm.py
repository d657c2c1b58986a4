"""Per-CTA timeline of k_spmm (JIGSAW_TRACE=1 + jigsaw_debug_trace) for a few
BASELINE shapes: where the microseconds of one launch go.  Developer tool."""
import os
import sys

import numpy as np

os.environ["JIGSAW_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402

NAMES = {1: "setup", 2: "A/E issued", 3: "B issued", 4: "1st stage full", 5: "last MMA commit",
         6: "acc ready", 7: "sends done", 8: "recv ready", 9: "stores done", 10: "exit sync",
         11: "dealloc", 16: "AE fetched", 17: "bar init done", 18: "fill decoded", 22: "B prefetch issued", 19: "B decoded",
         20: "G landed", 21: "MMA decoded", 23: "exit barrier"}


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x).view(np.int16)).cuda().view(torch.float16)


def report(tag, ev_us, tr, ghz):
    start, end = tr[:, 15], tr[:, 13]
    span = (end.max() - start.min()) / 1e3
    print(f"\n== {tag}: event {ev_us:.1f} us, CTA span {span:.1f} us, CTAs {len(tr)}, "
          f"start spread {(start.max() - start.min()) / 1e3:.2f} us, units/CTA min {tr[:, 12].min()} "
          f"median {int(np.median(tr[:, 12]))} max {tr[:, 12].max()}")
    last = (tr[:, 5] - tr[:, 0]) / ghz / 1e3
    last = np.where((last > 0) & (last < 1e4) & (tr[:, 8] > 0), last, 0)
    order = np.argsort(-last)[:8]
    print("   slowest CTAs (last MMA commit us, units, k-blocks, us waiting for data): " +
          ", ".join(f"#{i}: {last[i]:.1f} ({tr[i, 12]}, {tr[i, 8]}, {tr[i, 7] / ghz / 1e3:.1f})" for i in order))
    fast = np.argsort(last)
    fast = [i for i in fast if last[i] > 0][:4]
    print("   fastest CTAs: " + ", ".join(f"#{i}: {last[i]:.1f} ({tr[i, 12]}, {tr[i, 8]}, {tr[i, 7] / ghz / 1e3:.1f})"
                                         for i in fast))
    for k, name in NAMES.items():
        d = (tr[:, k] - tr[:, 0]) / ghz / 1e3
        d = d[(tr[:, k] != 0) & (d > -1) & (d < 1e4)]
        if len(d):
            print(f"   {name:16s} min {d.min():7.2f}  p10 {np.percentile(d, 10):7.2f}  median {np.median(d):7.2f}"
                  f"  p90 {np.percentile(d, 90):7.2f}  max {d.max():7.2f} us")


def main():
    torch.cuda.set_device(0)
    ghz = 1.965
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    pts = [(512, 2048, 2, 0.5, 256), (512, 2048, 8, 0.98, 256), (2048, 512, 4, 0.9, 256),
           (4096, 4096, 8, 0.9, 2048)]
    hs, Bs, Cs = [], [], []
    for i, (M, K, v, s, N) in enumerate(pts):
        A = synth.vector_sparse(M, K, v, s, i)
        h = jig.reorder(dev(A), v)
        B = dev(synth.dense_b(K, N, i))
        C = torch.empty((M, N), dtype=torch.float16, device="cuda")
        hs.append(h); Bs.append(B); Cs.append(C)
        for rep in range(3):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            h.spmm(B, C=C)
            e1.record()
            torch.cuda.synchronize()
        report(f"single {M}x{K} v{v} s{s} N{N}", e0.elapsed_time(e1) * 1e3, jig.debug_trace(), ghz)
    # grouped: the whole C2 batch
    mats = [(synth.vector_sparse(M, K, v, s, 50 + i), synth.dense_b(K, N, 50 + i), v)
            for i, (M, K, v, s, N) in enumerate(synth.c2_points())]
    hs2 = [jig.reorder(dev(a), v) for a, _, v in mats]
    B2 = [dev(b) for _, b, _ in mats]
    C2 = [torch.empty((a.shape[0], b.shape[1]), dtype=torch.float16, device="cuda") for a, b, _ in mats]
    for rep in range(3):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        jig.spmm_batched(hs2, B2, C2)
        e1.record()
        torch.cuda.synchronize()
    tr = jig.debug_trace()
    report("grouped C2 batch (36)", e0.elapsed_time(e1) * 1e3, tr, ghz)
    kb = np.zeros(8 * 6 * 32, np.int64)
    import ctypes
    jig.lib().jigsaw_debug_trace(kb.ctypes.data_as(ctypes.c_void_p), -1)
    kb = kb.reshape(8, 6, 32)
    for cta in range(2):
        t0 = tr[cta, 0]
        print(f"  CTA {cta} per k-block (us after entry): AE-issue / B-issue / full-seen / after-cp / after-mma / commit")
        for k in range(32):
            row = [(kb[cta, r, k] - t0) / ghz / 1e3 if kb[cta, r, k] > t0 else float('nan') for r in (0, 1, 2, 4, 5, 3)]
            print("   kb %2d  " % k + "  ".join(f"{x:7.2f}" for x in row))


if __name__ == "__main__":
    main()
