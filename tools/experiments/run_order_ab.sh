# A/B: PTE link/unlink memory-order variants (hit mode, M2r, resident collage), alternating
mkdir -p gpurun_out
for i in 1 2; do
  for v in default $VARIANTS; do
    if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
    echo "== $v round $i"
    AP_LIB_PATH=$L timeout 300 python tools/prof_hit.py 65536 8 | grep -E "tile|range"
    AP_LIB_PATH=$L timeout 300 python tools/prof_minor.py 2>&1 | tail -2
    AP_LIB_PATH=$L timeout 300 python tools/prof_collage.py 1048576 8 2>&1 | grep group
  done
done
