#!/bin/bash
# round 2 pass 5: "check at dereference" (lazy unlink) build: GPU suite,
# hit/deref/Fig.6 vs the previous eager build, resident collage aligned and
# unaligned (two-phase straddle pins)
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2_tests5.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_tests5.txt
for v in lazy lazym2p4 vC; do
  AP_LIB_PATH=build/variants/lib_$v.so AP_DEREF_GRIDS=148,296,592 AP_FIG6_TBS=148,296 timeout 400 python tools/exp_hit.py
done > gpurun_out/r2_exp_hit5.txt 2>&1
for v in lazy vC; do
  for st in 4096 3072; do
    echo "== $v stride $st"; AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_STRIDE=$st AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 4 8
  done
done > gpurun_out/r2_coll_res5.txt 2>&1
