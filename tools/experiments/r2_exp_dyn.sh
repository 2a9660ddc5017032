#!/bin/bash
mkdir -p gpurun_out
( for v in product dyn; do
  if [ $v = product ]; then L=""; else L=build/variants/lib_$v.so; fi
  echo "== $v"
  AP_LIB_PATH=$L AP_EXP_FRAMES=4096,64,96,148 AP_EXP_GRIDS=64,148 timeout 600 python tools/exp_c1.py
done
echo "== dynprof phases"
AP_LIB_PATH=build/variants/lib_dynprof.so AP_EXP_POINTS=64x64,64x148,4096x148 timeout 600 python tools/exp_fault_phases.py
) > gpurun_out/r2_dyn.txt 2>&1
