#!/bin/bash
# round 2 pass 3: whole GPU suite on the current build, then the deref
# instruction-diet variants (speculative load on/off)
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2_tests3.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_tests3.txt
for v in spec nospec; do
  AP_LIB_PATH=build/variants/lib_$v.so AP_DEREF_GRIDS=296,592 AP_FIG6_TBS=148,296 timeout 400 python tools/exp_hit.py
done > gpurun_out/r2_exp_hit3.txt 2>&1
