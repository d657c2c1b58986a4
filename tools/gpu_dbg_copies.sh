# e2e host-buffer path: the C2 batch of bench.py outside bench.py, whole and per product
mkdir -p gpurun_out
cat > /tmp/c2_pinned.py <<'PY'
import sys, numpy as np, torch, synth, bench, paper_conf_icpp_zhanglyfyllq24_b200 as jig
pts, _, _ = bench.workload("c2")
jobs = bench.local_jobs("c2", pts, 0, 1)
mats, hs = [], []
for ji, (M, K, v, s, N, seed, n0, n1) in enumerate(jobs):
    A = bench.make_a("c2", ji, M, K, v, s, seed); B = synth.dense_b(K, N, seed)
    mats.append((A, B)); hs.append(jig.reorder(torch.from_numpy(A.view(np.int16)).cuda().view(torch.float16), v))
print("B dtypes/shapes", {(B.dtype.str, B.flags.c_contiguous) for _, B in mats}, flush=True)
keep = [torch.from_numpy(B.view(np.int16)).pin_memory() for (_, B) in mats]
pin_B = [torch.from_numpy(B.view(np.int16)).pin_memory().numpy().view(np.uint16) for (_, B) in mats]
pin_C = [torch.empty((A.shape[0], B.shape[1]), dtype=torch.int16).pin_memory().numpy().view(np.uint16) for (A, B) in mats]
print("distinct B ptrs", len({p.ctypes.data for p in pin_B}), "of", len(pin_B), "base types", {type(p.base).__name__ for p in pin_B}, flush=True)
for tag, bl in [("temporaries", pin_B), ("kept tensors", [t.numpy().view(np.uint16) for t in keep])]:
    try:
        jig.spmm_batched_host(hs, bl, pin_C); print(tag, "whole batch ok", flush=True)
    except Exception as e:
        print(tag, "whole batch FAIL", e, flush=True)
PY
JIGSAW_DEBUG_COPIES=1 PYTHONPATH=$PWD timeout 300 python /tmp/c2_pinned.py 2>&1 | grep -v "^  "
