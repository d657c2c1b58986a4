mkdir -p gpurun_out
timeout 600 python tools/single_c2.py > gpurun_out/s15_single.txt 2>&1
