# PDL A/B: GPU tests, single-product graph timing with and without the
# programmatic-dependency launch attribute, default C2 bench line
mkdir -p gpurun_out
T=${1:-r01t}
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_gpu_tests.txt 2>&1
POINTS=0,8,9,10,15,16,26,27,33,34 REPS=3 timeout 600 python tools/single_c2.py > gpurun_out/${T}_single_pdl.txt 2>&1
JIGSAW_PDL=0 POINTS=0,8,9,10,15,16,26,27,33,34 REPS=3 timeout 600 python tools/single_c2.py > gpurun_out/${T}_single_nopdl.txt 2>&1
timeout 900 python bench.py --no-cpu > gpurun_out/${T}_bench_c2.json 2> gpurun_out/${T}_bench_c2.err
tail -3 gpurun_out/${T}_gpu_tests.txt
