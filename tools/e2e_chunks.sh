mkdir -p gpurun_out
T=$1
for c in 1 3 6 12; do for w in c2 c4; do
  v=$(JIGSAW_HOST_CHUNKS=$c timeout 400 python bench.py --workload $w --no-cpu --no-cublas --steps 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['e2e']['value'],1))")
  echo "chunks=$c $w e2e $v TF/s" >> gpurun_out/${T}_e2e.txt
done; done
