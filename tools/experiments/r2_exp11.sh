#!/bin/bash
# round 2 pass 11: C1 with one walking pointer per warp (drop-behind can see
# the page left behind), fault path at 64 vs 128 registers; hit mode check
mkdir -p gpurun_out
for v in s64 s128; do
  echo "== $v"
  AP_LIB_PATH=build/variants/lib_$v.so python bench.py --workload c1 --steps 5 --warmup 3 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], json.dumps(d['fault_bound']))"
  AP_LIB_PATH=build/variants/lib_$v.so python bench.py --workload c3 --steps 2 --warmup 1 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c3', d['value'], d['ms_per_step'])"
  AP_LIB_PATH=build/variants/lib_$v.so AP_DEREF_GRIDS=148 AP_FIG6_TBS=148 timeout 400 python tools/exp_hit.py | grep -E "tile|range|deref|16B (read|add)"
  AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 8
done > gpurun_out/r2_c1_11.txt 2>&1
