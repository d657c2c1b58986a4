mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "pair" 2>&1 | tail -25 > gpurun_out/pair_tests.txt
cat gpurun_out/pair_tests.txt
for wl in c2 c4; do for pr in 128 256; do
timeout 300 python bench.py --workload $wl --panel-rows $pr --steps 50 --warmup 5 --no-cpu > gpurun_out/pair_${wl}_${pr}.json 2> gpurun_out/pair_${wl}_${pr}.err
python -c "import json;d=json.load(open('gpurun_out/pair_${wl}_${pr}.json'));print('$wl','$pr',d['value'],d['ms_per_step'],d['roofline']['frac'],d['cublas']['speedup_step'])"
done; done
