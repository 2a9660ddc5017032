#!/bin/bash
# unaligned collage: both pages linked at once (split) vs lmhoist; C5/C4u vs the pre-C1-change build
mkdir -p gpurun_out
( for v in lmhoist split; do
  echo "== $v"; AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 8 | grep N=
  AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_STRIDE=3072 AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 4 8 16 | grep N=
done
timeout 900 python -m pytest tests/test_gpu_collage.py -x -q 2>&1 | tail -2
for v in pre split pre split; do
  echo "== c4u/c5 $v"
  AP_LIB_PATH=build/variants/lib_$v.so timeout 900 python bench.py --workload c4 --stride 3072 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c4u', d['value'], d['roofline']['frac'])"
  AP_LIB_PATH=build/variants/lib_$v.so timeout 900 python bench.py --workload c5 --steps 3 --warmup 2 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c5', d['value'], d['roofline']['frac'])"
done ) > gpurun_out/r2_split.txt 2>&1
