#!/bin/bash
# Round-2 GPU evidence (run under gpurun): default bench line, reference arm,
# C5 sweep at N = 1, ncu launch list of a short bench, ncu --set full of the C2
# and C4 grouped k_spmm launches.  Outputs in gpurun_out/ with prefix $1.
P=${1:-r02}
python bench.py > gpurun_out/${P}_bench_default.json 2> gpurun_out/${P}_bench_default.err
python bench.py --impl reference > gpurun_out/${P}_bench_reference.json 2> gpurun_out/${P}_bench_reference.err
python bench.py --multi --no-cublas --no-extra --no-cpu --steps 10 > gpurun_out/${P}_bench_multi_n1.json 2> gpurun_out/${P}_bench_multi_n1.err
# launch list of the timed steps only (bench.py brackets them with
# cudaProfilerStart/Stop when BENCH_CUDA_PROFILER=1)
BENCH_CUDA_PROFILER=1 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${P}_launches_c2.csv \
    python bench.py --steps 5 --warmup 3 --no-cpu --no-cublas --no-extra > /dev/null 2>&1
BENCH_CUDA_PROFILER=1 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${P}_launches_c4.csv \
    python bench.py --workload c4 --steps 5 --warmup 3 --no-cpu --no-cublas > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 2 -c 1 -o gpurun_out/${P}_c2_grouped \
    python tools/ncu_one.py c2 > gpurun_out/${P}_ncu_c2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 2 -c 1 -o gpurun_out/${P}_c4 \
    python tools/ncu_one.py c4 > gpurun_out/${P}_ncu_c4.log 2>&1
