#!/bin/bash
mkdir -p gpurun_out
for v in cc6 cc12m3 cc12m2 cc16m3 cc24m2; do
  echo "== $v"; AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 2 4 8 16 | grep N=
  AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_STRIDE=3072 AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 8 16 | grep N=
  AP_LIB_PATH=build/variants/lib_$v.so timeout 600 python bench.py --workload c4 --steps 3 --warmup 2 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('cold c4', d['value'], d['collage']['fill_GB'])"
done > gpurun_out/r2_ch21.txt 2>&1
