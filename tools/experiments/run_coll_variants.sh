# collage on a resident cache: library variants (build/variants/lib_*.so) vs the default
mkdir -p gpurun_out
for v in default $(ls build/variants 2>/dev/null | sed -n 's/^lib_\(.*\)\.so$/\1/p'); do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
  echo "== $v"; AP_LIB_PATH=$L timeout 300 python tools/prof_collage.py 1048576 ${GROUPS_:-1 4}
done > gpurun_out/coll_variants.txt 2>&1
cat gpurun_out/coll_variants.txt
