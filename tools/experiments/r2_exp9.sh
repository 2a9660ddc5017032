#!/bin/bash
# round 2 pass 9: pipelined collage translation, occupancy variants: resident
# (aligned + unaligned) and cold C4
mkdir -p gpurun_out
for v in cnp cp4 cp3 cp2; do
  for st in 4096 3072; do
    echo "== $v stride $st"; AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_STRIDE=$st AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 4 8
  done
  echo "== $v cold C4"; AP_LIB_PATH=build/variants/lib_$v.so timeout 600 python bench.py --workload c4 --steps 3 --warmup 2 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['value'], d['collage']['fill_GB'], d['collage'].get('resident_cache',{}).get('group8'))"
done > gpurun_out/r2_coll_pipe9.txt 2>&1
