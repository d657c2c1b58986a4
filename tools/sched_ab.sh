# C2 with 256-row panels: static pair schedule under different per-unit costs
mkdir -p gpurun_out
T=$1
for nt in 256 128; do for uc in 1 3 6; do
  v=$(JIGSAW_FORCE_NT=$nt JIGSAW_UNIT_COST=$uc timeout 300 python bench.py --panel-rows 256 --no-cpu --no-cublas --steps 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['roofline']['per_launch_us'],1))")
  echo "P256 NT=$nt unit_cost=$uc: $v us" >> gpurun_out/${T}_sched.txt
done; done
JIGSAW_DEBUG_SCHED=1 JIGSAW_FORCE_NT=256 timeout 300 python bench.py --panel-rows 256 --no-cpu --no-cublas --steps 3 2>&1 >/dev/null | grep "pair schedule" | head -2 >> gpurun_out/${T}_sched.txt
