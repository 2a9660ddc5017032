#!/bin/bash
mkdir -p gpurun_out
( for v in pipe2 pipe1 pipe2; do
  echo "== $v"; AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 4 8 | grep N=
done
echo "== product"; AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 4 8 | grep N=
AP_LIB_PATH=build/variants/lib_pipe2.so timeout 600 python bench.py --workload c4 --steps 3 --warmup 2 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('pipe2 cold c4', d['value'])"
AP_LIB_PATH=build/variants/lib_pipe2.so timeout 900 python -m pytest tests/test_gpu_collage.py -x -q 2>&1 | tail -1
) > gpurun_out/r2_pipe2.txt 2>&1
