#!/bin/bash
mkdir -p gpurun_out
( timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for v in pre lean2 pre lean2; do
  echo "== $v"; AP_LIB_PATH=build/variants/lib_$v.so AP_DEREF_GRIDS=148 AP_FIG6_TBS=148 timeout 400 python tools/exp_hit.py | grep -E "tile|deref|read|add|reduce"
done
echo "== lean2 collage"; AP_LIB_PATH=build/variants/lib_lean2.so AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 4 8 | grep N=
AP_LIB_PATH=build/variants/lib_lean2.so AP_PROF_STRIDE=3072 AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 4 8 16 | grep N=
timeout 600 python bench.py --workload c1 --steps 5 --warmup 3 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c1', d['value'], d['roofline']['frac'])"
) > gpurun_out/r2_lean2.txt 2>&1
