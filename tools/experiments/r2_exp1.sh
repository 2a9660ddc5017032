#!/bin/bash
# round 2, first GPU pass: GPU tests on the ABI-call (rdc) build, then the
# hit-regime / Fig. 6 A/B over library variants (round-1 build vs rdc builds
# with per-access pipeline depth 1/2/4/8).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2_smi.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r2_tests1.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_tests1.txt
for v in r1 p1 p2 p4 p8; do
  AP_LIB_PATH=build/variants/lib_$v.so AP_DEREF_GRIDS=148,296,592 timeout 400 python tools/exp_hit.py
done > gpurun_out/r2_exp_hit1.txt 2>&1
