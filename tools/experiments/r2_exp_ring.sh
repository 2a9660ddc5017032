#!/bin/bash
# drop-behind ring: GPU tests touching the policies/invariants, C1 sweeps, fault phases
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_reads.py tests/test_gpu_stress.py -x -q > gpurun_out/r2_ring_tests.txt 2>&1
tail -2 gpurun_out/r2_ring_tests.txt
AP_EXP_FRAMES=4096,64,65,96,128,148 AP_EXP_GRIDS=64,148,296 timeout 600 python tools/exp_c1.py > gpurun_out/r2_ring_c1.txt 2>&1
AP_LIB_PATH=build/variants/lib_fprof.so timeout 600 python tools/exp_fault_phases.py > gpurun_out/r2_ring_phases.txt 2>&1
timeout 600 python bench.py --workload c1 --steps 5 --warmup 3 > gpurun_out/r2_ring_bench_c1.json 2> gpurun_out/r2_ring_bench_c1.err
