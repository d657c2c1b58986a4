for rep in 1 2; do
  for lib in prev new; do
    if [ $lib = new ]; then unset JIGSAW_LIB_AB; else export JIGSAW_LIB_AB=tools/libjigsaw_$lib.so; fi
    python tools/probe_c2_cfg.py c2 0 0 $lib
    python tools/probe_c2_cfg.py c4 0 0 $lib
    python tools/probe_c2_cfg.py c3 0 0 $lib
  done
done
