P=tools/probe_c2_cfg.py
python $P c4 0 0 c4_nt256
python $P c4 0 128 c4_nt128
python $P c4 128 0 c4_p128_auto
python $P c5b 0 0 c5b_nt256
python $P c5b 0 128 c5b_nt128
