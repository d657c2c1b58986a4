mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/s1_smi.txt 2>&1
timeout 900 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -15 > gpurun_out/s1_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s1_smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/s1_bench_default.json 2> gpurun_out/s1_bench_default.err
timeout 600 python bench.py --workload c4 > gpurun_out/s1_bench_c4.json 2> gpurun_out/s1_bench_c4.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/s1_ref.json 2> gpurun_out/s1_ref.err
