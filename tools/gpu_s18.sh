mkdir -p gpurun_out
for h in 0 1 2 3 7; do for wl in c4 c2; do
JIGSAW_L2HINTS=$h timeout 300 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu --no-cublas > /tmp/b.json 2>/dev/null
python -c "import json;b=json.load(open('/tmp/b.json'));print('hints $h $wl',round(b['value'],1),round(b['ms_per_step']*1e3,1),'us')" >> gpurun_out/s18_hints.txt
done; done
