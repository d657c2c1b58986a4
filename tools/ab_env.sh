# A/B an environment switch on the C2 / C4 grouped launches (tools/time_c2.py style timing)
# usage: tools/ab_env.sh "ENV=1" [workloads]
for wl in ${2:-c2 c4}; do
  timeout 300 python bench.py --workload $wl --steps 30 --warmup 5 --no-cpu --no-cublas > /tmp/a.json 2>/dev/null
  env $1 timeout 300 python bench.py --workload $wl --steps 30 --warmup 5 --no-cpu --no-cublas > /tmp/b.json 2>/dev/null
  python -c "import json;a=json.load(open('/tmp/a.json'));b=json.load(open('/tmp/b.json'));print('$wl','default',round(a['ms_per_step']*1e3,1),'us','| $1',round(b['ms_per_step']*1e3,1),'us')"
done
