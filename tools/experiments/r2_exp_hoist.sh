#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2_hoist_tests.txt 2>&1
tail -2 gpurun_out/r2_hoist_tests.txt
( AP_EXP_PATTERN=3 AP_EXP_FRAMES=4096,64,96 AP_EXP_GRIDS=64,148 timeout 600 python tools/exp_c1.py
  echo "== phases queue"; AP_EXP_PATTERN=3 AP_LIB_PATH=build/variants/lib_fprof.so AP_EXP_POINTS=4096x64,64x64,64x148 timeout 600 python tools/exp_fault_phases.py ) > gpurun_out/r2_hoist_c1.txt 2>&1
timeout 600 python bench.py --workload c1 --steps 5 --warmup 3 > gpurun_out/r2_hoist_bench_c1.json 2> gpurun_out/r2_hoist_bench_c1.err
timeout 900 python bench.py --steps 5 --warmup 3 --no-collage --no-cpu-baseline > gpurun_out/r2_hoist_bench_c2.json 2> gpurun_out/r2_hoist_bench_c2.err
