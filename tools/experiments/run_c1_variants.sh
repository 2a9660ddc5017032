# C1 under back-off / sweep settings, default library vs variants
for v in default ${VARIANTS}; do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
  echo "== $v"; AP_LIB_PATH=$L timeout 300 python tools/c1_backoff.py
done
