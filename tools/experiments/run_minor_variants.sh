for i in 1 2; do for v in default $VARIANTS; do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
  echo -n "$v: "; AP_LIB_PATH=$L timeout 300 python tools/prof_minor.py 2>&1 | tail -1
done; done
