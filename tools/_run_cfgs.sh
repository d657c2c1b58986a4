P=tools/probe_c2_cfg.py
for r in 1 2; do
python abold/probe_old.py c2
python $P c2 0 0 new_c2
python abold/probe_old.py c4
python $P c4 0 0 new_c4
done
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv
