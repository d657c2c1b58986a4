mkdir -p gpurun_out
timeout 300 python tools/single_c2.py > gpurun_out/s2_single_events.txt 2>&1
REPS=2 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_single_ncu.csv python tools/single_c2.py > gpurun_out/s2_single_ncu.log 2>&1
timeout 300 python tools/trace_spmm.py > gpurun_out/s2_trace.txt 2>&1
