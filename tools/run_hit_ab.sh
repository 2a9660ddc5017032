# hit-mode A/B: default library vs build/variants/lib_old.so, alternating, 3 rounds
for i in 1 2 3; do
  for v in default old; do
    if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
    echo -n "$v: "; AP_LIB_PATH=$L timeout 300 python tools/prof_hit.py 65536 8 | grep tile
  done
done
for i in 1 2; do
  for v in default old; do
    if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
    echo "$v: "; AP_LIB_PATH=$L timeout 300 python tools/prof_collage.py 1048576 8 | grep group
  done
done
for v in default old; do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
  AP_LIB_PATH=$L timeout 600 python bench.py --workload c4 --no-cpu-baseline --steps 3 > gpurun_out/ab_c4_$v.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/ab_c4_$v.json'));print('$v c4', d['value'], d['collage']['major_faults'], d['collage']['resident_cache']['group8'])"
done
