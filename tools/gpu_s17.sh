mkdir -p gpurun_out
for sched in lpt loc; do for wl in c4 c2; do
JIGSAW_SCHED=$sched timeout 300 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu --no-cublas > /tmp/b.json 2>/dev/null
python -c "import json;b=json.load(open('/tmp/b.json'));print('$sched $wl',round(b['value'],1),round(b['ms_per_step']*1e3,1),'us')" >> gpurun_out/s17_sched.txt
done; done
JIGSAW_SCHED=loc timeout 600 ncu --set full --clock-control none -k regex:k_spmm -s 2 -c 1 -o gpurun_out/s17_c4_loc python tools/run_c2_batch.py c4 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:k_spmm -s 2 -c 1 -o gpurun_out/s17_c4_lpt python tools/run_c2_batch.py c4 > /dev/null 2>&1
