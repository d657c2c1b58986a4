"""End-to-end host-buffer path (jigsaw_spmm_batched_host) of the C2 batch against
its PCIe floor on the same box: the same bytes copied H2D and D2H from / to
pinned memory (one copy per direction, and in 16 chunks on two streams), and
the call at several chunk counts.  Developer tool."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_icpp_zhanglyfyllq24_b200 as jig  # noqa: E402


def wall(fn, n=20, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(n):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / n * 1e3


def main():
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    name = sys.argv[1] if len(sys.argv) > 1 else "c2"
    b = bench.Batch(name, 0, 1, 0, dev, torch, jig)
    nb = sum(B.size for (_, B) in b.mats)
    nc = sum(M * N for (M, K, v, s, N) in b.points)
    hb = torch.empty(nb, dtype=torch.int16).pin_memory()
    hc = torch.empty(nc, dtype=torch.int16).pin_memory()
    db = torch.empty(nb, dtype=torch.int16, device=dev)
    dc = torch.empty(nc, dtype=torch.int16, device=dev)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def copies_one():
        with torch.cuda.stream(s1):
            db.copy_(hb, non_blocking=True)
        with torch.cuda.stream(s2):
            hc.copy_(dc, non_blocking=True)
        s1.synchronize()
        s2.synchronize()

    def copies_chunked(k=16):
        eb = [(i * nb) // k for i in range(k + 1)]
        ec = [(i * nc) // k for i in range(k + 1)]
        for i in range(k):
            with torch.cuda.stream(s1):
                db[eb[i]:eb[i + 1]].copy_(hb[eb[i]:eb[i + 1]], non_blocking=True)
            with torch.cuda.stream(s2):
                hc[ec[i]:ec[i + 1]].copy_(dc[ec[i]:ec[i + 1]], non_blocking=True)
        s1.synchronize()
        s2.synchronize()

    out = {"workload": name, "MB_each_way": [2 * nb / 1e6, 2 * nc / 1e6]}
    out["h2d_only_ms"] = wall(lambda: (db.copy_(hb, non_blocking=True), torch.cuda.synchronize()))
    out["d2h_only_ms"] = wall(lambda: (hc.copy_(dc, non_blocking=True), torch.cuda.synchronize()))
    out["both_one_copy_each_ms"] = wall(copies_one)
    out["both_16_chunks_ms"] = wall(copies_chunked)
    pin_B, pin_C, ob, oc = [], [], 0, 0
    hbn, hcn = hb.numpy().view(np.uint16), hc.numpy().view(np.uint16)
    for (_, B), (M, K, v, s, N) in zip(b.mats, b.points):
        pin_B.append(hbn[ob:ob + B.size].reshape(B.shape))
        pin_B[-1][...] = B
        pin_C.append(hcn[oc:oc + M * N].reshape(M, N))
        ob += B.size
        oc += M * N
    for ch in (0, 4, 8, 16, 32):
        jig.set_launch_override(host_chunks=ch)
        out[f"e2e_chunks_{ch or 'default'}_ms"] = wall(lambda: jig.spmm_batched_host(b.hs, pin_B, pin_C))
    jig.set_launch_override()
    # the same call through the C ABI directly (ctypes arrays built once): the
    # binding's per-call Python work is the difference
    import ctypes
    n = len(b.hs)
    hsa = (ctypes.c_void_p * n)(*[h.ptr.value for h in b.hs])
    bpa = (ctypes.c_void_p * n)(*[x.ctypes.data for x in pin_B])
    cpa = (ctypes.c_void_p * n)(*[x.ctypes.data for x in pin_C])
    nsa = (ctypes.c_int64 * n)(*[x.shape[1] for x in pin_B])
    L = jig.lib()
    out["e2e_direct_abi_ms"] = wall(lambda: L.jigsaw_spmm_batched_host(hsa, bpa, nsa, cpa, n, None))
    t0 = time.perf_counter()
    for _ in range(200):
        jig._host16(pin_B[0], "B")
    out["host16_us"] = (time.perf_counter() - t0) / 200 * 1e6
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
