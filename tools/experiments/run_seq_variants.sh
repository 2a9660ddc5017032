# hit-mode SEQ kernels: library variants lib_m<minb>t<tile>.so at grid 148*minb, 2 rounds
for i in 1 2; do
for v in default $(ls build/variants 2>/dev/null | sed -n 's/^lib_\(.*\)\.so$/\1/p'); do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; n=1; else L=build/variants/lib_$v.so; n=${v:1:1}; fi
  echo -n "$v grid $((148*n)): "; AP_GRID=$((148*n)) AP_LIB_PATH=$L timeout 300 python tools/prof_hit.py 65536 8 | grep -E "tile|range" | tr '\n' ' '; echo
done
done
