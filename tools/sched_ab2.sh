# per-unit cost sweep: C2 with 256-row panels (NT=256 static pair schedule) and 128-row panels (dynamic)
mkdir -p gpurun_out
T=$1
for uc in 4 6 8 10 14; do
  v=$(JIGSAW_FORCE_NT=256 JIGSAW_UNIT_COST=$uc timeout 300 python bench.py --panel-rows 256 --no-cpu --no-cublas --steps 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['roofline']['per_launch_us'],1))")
  echo "C2 P256 NT=256 unit_cost=$uc: $v us" >> gpurun_out/${T}_sched.txt
  JIGSAW_DEBUG_SCHED=1 JIGSAW_FORCE_NT=256 JIGSAW_UNIT_COST=$uc timeout 300 python bench.py --panel-rows 256 --no-cpu --no-cublas --steps 3 2>&1 >/dev/null | grep "pair schedule" | head -1 >> gpurun_out/${T}_sched.txt
done
for uc in 1 3 6; do
  v=$(JIGSAW_UNIT_COST=$uc timeout 300 python bench.py --panel-rows 128 --no-cpu --no-cublas --steps 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['roofline']['per_launch_us'],1))")
  echo "C2 P128 unit_cost=$uc: $v us" >> gpurun_out/${T}_sched.txt
done
for uc in 1 3 6; do
  v=$(JIGSAW_UNIT_COST=$uc timeout 300 python bench.py --workload c4 --no-cpu --no-cublas --steps 30 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['roofline']['per_launch_us'],1))")
  echo "C4 auto unit_cost=$uc: $v us" >> gpurun_out/${T}_sched.txt
done
