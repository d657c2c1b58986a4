# quick device-time numbers of the grouped C2 / C4 steps at both panel heights
for wl in ${1:-c2 c4}; do for pr in 128 256; do
timeout 300 python bench.py --workload $wl --panel-rows $pr --steps 30 --warmup 5 --no-cpu --no-cublas > /tmp/q.json 2>/dev/null
python -c "import json;d=json.load(open('/tmp/q.json'));print('$wl P=$pr',round(d['value'],1),'TF/s',round(d['ms_per_step']*1e3,1),'us')"
done; done
