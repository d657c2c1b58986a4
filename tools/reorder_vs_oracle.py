"""GPU reorder throughput against the CPU oracle's reorder, side
by side on the same box, for the C2 matrices (and the C1 case): oracle.reorder
(plain C, one thread) wall time vs jigsaw_reorder device time (min of 3 builds),
and bit-identity of the two formats.  Developer tool; one JSON line per matrix."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402


def main():
    torch.cuda.set_device(0)
    pts = [(256, 256, 4, 0.8, 64)] + list(synth.c2_points())
    tot_cpu = tot_gpu = 0.0
    for i, (M, K, v, s, N) in enumerate(pts):
        A = synth.vector_sparse(M, K, v, s, 700 + i)
        t0 = time.perf_counter()
        ref = oracle.reorder(A, P=128)
        cpu_ms = (time.perf_counter() - t0) * 1e3
        a = torch.from_numpy(A.view(np.int16)).cuda().view(torch.float16)
        ms = []
        for rep in range(3):
            h = jig.reorder(a, v)
            ms.append(h.info()["reorder_ms"])
            if rep < 2:
                h.free()
        g = h.export()
        same = bool(np.array_equal(g["T"], ref.T) and np.array_equal(g["col_idx"], ref.col_idx)
                    and np.array_equal(g["perm"], ref.perm) and np.array_equal(g["vals"], ref.vals)
                    and np.array_equal(g["meta"], ref.meta))
        h.free()
        tot_cpu += cpu_ms
        tot_gpu += min(ms)
        print(json.dumps({"M": M, "K": K, "v": v, "s": s, "tiles": int(ref.T.sum()), "cpu_oracle_ms": cpu_ms,
                          "gpu_device_ms": min(ms), "speedup": cpu_ms / min(ms), "bit_identical": same}), flush=True)
    print(json.dumps({"total_cpu_oracle_ms": tot_cpu, "total_gpu_device_ms": tot_gpu, "speedup": tot_cpu / tot_gpu,
                      "cpu_threads": 1}), flush=True)


if __name__ == "__main__":
    main()
