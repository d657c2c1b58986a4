mkdir -p gpurun_out
JIGSAW_NO_PREFETCH=1 timeout 300 python tools/trace_single.py > gpurun_out/s6_trace_single_nopf.txt 2>&1
