#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_reads.py tests/test_gpu_stress.py tests/test_gpu_writes.py tests/test_gpu_compute.py -x -q > gpurun_out/r2_pin_tests.txt 2>&1
tail -2 gpurun_out/r2_pin_tests.txt
( for pat in 0 3; do echo "== pattern $pat"; AP_EXP_PATTERN=$pat AP_EXP_FRAMES=4096,64,96,148 AP_EXP_GRIDS=64,148 timeout 600 python tools/exp_c1.py; done
  echo "== phases queue"; AP_EXP_PATTERN=3 AP_LIB_PATH=build/variants/lib_fprof.so AP_EXP_POINTS=4096x64,64x64,64x148,4096x148 timeout 600 python tools/exp_fault_phases.py ) > gpurun_out/r2_pin_c1.txt 2>&1
timeout 600 python bench.py --workload c1 --steps 5 --warmup 3 > gpurun_out/r2_pin_bench_c1.json 2> gpurun_out/r2_pin_bench_c1.err
