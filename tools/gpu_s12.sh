mkdir -p gpurun_out
timeout 600 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -5 > gpurun_out/s12_tests.txt
timeout 300 python tools/trace_single.py > gpurun_out/s12_trace_single.txt 2>&1
timeout 300 python tools/single_c2.py > gpurun_out/s12_single_events.txt 2>&1
timeout 300 python bench.py --steps 50 --warmup 5 --no-cpu > gpurun_out/s12_bench_c2.json 2> gpurun_out/s12_bench_c2.err
