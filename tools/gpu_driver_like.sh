# what the driver runs at round end: GPU suite, smoke, default bench, reference arm (timed by wall clock)
mkdir -p gpurun_out
T=${1:-x}
timeout 900 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -3 | tee gpurun_out/${T}_gpu_tests.txt
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
s=$(date +%s); timeout 900 python bench.py > gpurun_out/${T}_bench_default.json 2> gpurun_out/${T}_bench_default.err; echo "bench wall $(( $(date +%s) - s )) s"
s=$(date +%s); timeout 900 python bench.py --impl reference > gpurun_out/${T}_bench_ref_default.json 2>/dev/null; echo "reference wall $(( $(date +%s) - s )) s"
python -c "import json;d=json.load(open('gpurun_out/${T}_bench_default.json'));print({k:d[k] for k in ['value','ms_per_step','e2e','gpu_launches','clocks']}, d['roofline']['frac'])"
