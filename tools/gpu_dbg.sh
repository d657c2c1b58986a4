# C4 data-movement ceiling per variant: normal vs JIGSAW_DBG=2 (MMAs skipped; timing only)
mkdir -p gpurun_out
TAG=$1; shift
for defs in "$@"; do
  JIGSAW_NVCC_DEFINES="$defs" python -c "from paper_conf_icpp_zhanglyfyllq24_b200 import _build; _build.build(force=True)" || continue
  for dbg in 0 2; do
    JIGSAW_DBG=$dbg timeout 300 python bench.py --workload c4 --steps 10 --warmup 3 --no-cpu --no-cublas > /tmp/c4.json 2>/dev/null
    python -c "import json;b=json.load(open('/tmp/c4.json'));print('$defs dbg=$dbg C4',round(b['ms_per_step']*1e3,1),'us')" >> gpurun_out/${TAG}_dbg.txt 2>&1
  done
done
python -c "from paper_conf_icpp_zhanglyfyllq24_b200 import _build; _build.build(force=True)"
