# A/B of two library builds on one box: bench C2 (and optionally C4) short runs, interleaved
mkdir -p gpurun_out
T=$1; shift
for rep in 1 2; do
  for lib in "$@"; do
    for w in ${WORKLOADS:-c2}; do
      v=$(JIGSAW_LIB_AB=$lib timeout 300 python bench.py --workload $w --no-cpu --no-cublas --steps 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['roofline']['per_launch_us'],1))")
      echo "$lib $w rep$rep: $v us per launch" >> gpurun_out/${T}_ab.txt
    done
  done
done
