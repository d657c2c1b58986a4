# host-buffer pipeline: one vs two copy lanes per direction (e2e through jigsaw_spmm_batched_host)
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -q -k "batched_host" 2>&1 | tail -2
for rep in 1 2; do for wl in c2 c4; do for L in 1 2; do
JIGSAW_HOST_LANES=$L timeout 300 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu --no-cublas > gpurun_out/lanes_${wl}_$L.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/lanes_${wl}_$L.json'));print('$wl lanes=$L rep $rep e2e',round(d['e2e']['value'],2),'value',round(d['value'],1))"
done; done; done
