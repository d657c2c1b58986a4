# prologue restructure: GPU tests, trace of single products, single-product graph timing
mkdir -p gpurun_out
T=${1:-r01t2}
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_gpu_tests.txt 2>&1
timeout 300 python tools/trace_single.py > gpurun_out/${T}_trace_single.txt 2>&1
POINTS=0,8,9,10,15,16,26,27,33,34 REPS=3 timeout 600 python tools/single_c2.py > gpurun_out/${T}_single.txt 2>&1
tail -3 gpurun_out/${T}_gpu_tests.txt
