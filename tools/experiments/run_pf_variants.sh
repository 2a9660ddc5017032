# per-access (deref) hit read and Fig. 6 read/add with stride-prefetch variants lib_pf<dist>.so
for v in default pf2 pf4 pf8 pf16; do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
  for g in 148 592; do echo "== $v grid $g"; AP_GRID=$g AP_LIB_PATH=$L timeout 300 python tools/prof_hit.py 65536 4 | grep deref; done
done
