for r in 1 2; do
JIGSAW_LIB_AB=abprev/paper_conf_icpp_zhanglyfyllq24_b200/libjigsaw.so python tools/probe_c2_cfg.py c2 0 0 prevlib_c2
JIGSAW_LIB_AB=tools/libjigsaw_v7.so python tools/probe_c2_cfg.py c2 0 0 v7_c2
JIGSAW_LIB_AB=abprev/paper_conf_icpp_zhanglyfyllq24_b200/libjigsaw.so python tools/probe_c2_cfg.py c4 0 0 prevlib_c4
JIGSAW_LIB_AB=tools/libjigsaw_v7.so python tools/probe_c2_cfg.py c4 0 0 v7_c4
done
