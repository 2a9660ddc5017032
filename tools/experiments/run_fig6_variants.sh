# Fig. 6 sweep + per-access hit read for library variants lib_m<compute minb>d<deref minb>.so
for v in m1d2 m2d3 m3d4; do
 m=${v:1:1}; d=${v:3:1}
 echo "=== $v compute minb $m"; AP_FIG6_MINB=$m AP_LIB_PATH=build/variants/lib_$v.so timeout 300 python tools/fig6_sweep.py
 echo "=== deref minb $d grid $((148*d))"; AP_GRID=$((148*d)) AP_LIB_PATH=build/variants/lib_$v.so timeout 300 python tools/prof_hit.py 65536 4 | grep deref
done
