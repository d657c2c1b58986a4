# full GPU test suite + C2 / C4 benches at both panel heights (no cuBLAS / CPU legs)
mkdir -p gpurun_out
TAG=${1:-x}
timeout 900 python -m pytest tests/ -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} 2>&1 | tail -15 > gpurun_out/${TAG}_tests.txt
cat gpurun_out/${TAG}_tests.txt
for wl in c2 c4; do for pr in 128 256; do
timeout 300 python bench.py --workload $wl --panel-rows $pr --steps 50 --warmup 5 --no-cpu --no-cublas > gpurun_out/${TAG}_${wl}_${pr}.json 2> gpurun_out/${TAG}_${wl}_${pr}.err
python -c "import json;d=json.load(open('gpurun_out/${TAG}_${wl}_${pr}.json'));print('$wl P=$pr',round(d['value'],1),round(d['ms_per_step']*1e3,1),'us frac',round(d['roofline']['frac'],3))" || tail -5 gpurun_out/${TAG}_${wl}_${pr}.err
done; done
