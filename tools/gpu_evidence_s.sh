# round evidence: default bench line (C2, with cuBLAS + CPU legs), C4 line, reference arm,
# ncu launch list of the default bench, ncu --set full of the grouped C2 and C4 k_spmm launches,
# single-product graph timing, and an NT=256 A/B for C2
mkdir -p gpurun_out
T=${1:-r01s}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${T}_smi.txt 2>&1
timeout 900 python bench.py > gpurun_out/${T}_bench_c2.json 2> gpurun_out/${T}_bench_c2.err
timeout 900 python bench.py --workload c4 > gpurun_out/${T}_bench_c4.json 2> gpurun_out/${T}_bench_c4.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${T}_bench_ref.json 2> gpurun_out/${T}_bench_ref.err
JIGSAW_FORCE_NT=256 timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu --no-cublas > gpurun_out/${T}_c2_nt256.json 2>/dev/null
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/${T}_ncu_launches_c2.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-cublas > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 2 -c 1 \
   -o gpurun_out/${T}_c2_grouped python tools/run_c2_batch.py > gpurun_out/${T}_ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 2 -c 1 \
   -o gpurun_out/${T}_c4 python tools/run_c2_batch.py c4 > gpurun_out/${T}_ncu_c4.log 2>&1
timeout 600 python tools/single_c2.py > gpurun_out/${T}_single.txt 2>&1
ls -la gpurun_out | grep $T
