for w in c3 venom c1 c5a c5b; do python bench.py --workload $w --no-cpu --steps 20 > gpurun_out/r02fs_bench_$w.json 2> gpurun_out/r02fs_bench_$w.err; done
python bench.py --workload c2 --panel-rows 256 --no-cpu --no-extra --steps 20 > gpurun_out/r02fs_bench_c2_p256.json 2> gpurun_out/r02fs_bench_c2_p256.err
