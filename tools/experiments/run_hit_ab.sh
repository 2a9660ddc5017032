# A/B: default library vs build/variants/lib_old.so (hit mode, M2r, resident collage), alternating
for i in 1 2 3; do
  for v in default old; do
    if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
    echo -n "$v: "; AP_LIB_PATH=$L timeout 300 python tools/prof_hit.py 65536 8 | grep -E "tile|range" | tr '\n' ' '; echo
  done
done
for v in default old; do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
  echo -n "$v M2r: "; AP_LIB_PATH=$L timeout 300 python tools/prof_minor.py
  echo "$v collage: "; AP_LIB_PATH=$L timeout 300 python tools/prof_collage.py 1048576 8 | grep group
done
