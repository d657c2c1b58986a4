# host-buffer pipeline: per-chunk segment-copy kernel over mapped pinned memory vs one cudaMemcpyAsync per product
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "batched_host or threads" 2>&1 | tail -2
for rep in 1 2; do for wl in c2 c4; do for K in 0 1; do
JIGSAW_HOST_COPY_KERNEL=$K timeout 300 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu --no-cublas > gpurun_out/ck_${wl}_$K.json 2>gpurun_out/ck_${wl}_$K.err
python -c "import json;d=json.load(open('gpurun_out/ck_${wl}_$K.json'));print('$wl copy_kernel=$K rep $rep e2e',round(d['e2e']['value'],2),'value',round(d['value'],1))" || tail -2 gpurun_out/ck_${wl}_$K.err
done; done; done
