mkdir -p gpurun_out
timeout 300 python tools/trace_single.py > gpurun_out/s13_trace_single.txt 2>&1
