P=tools/probe_c2_cfg.py
for w in c2 c4 c3 c5a; do python $P $w 0 0 ${w}_static; done
