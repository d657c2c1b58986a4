mkdir -p gpurun_out
timeout 300 python tools/trace_single.py > gpurun_out/s3_trace_single.txt 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/mc_bench tools/mc_bench.cu -lcuda && timeout 120 /tmp/mc_bench > gpurun_out/s3_mc_bench.txt 2>&1
