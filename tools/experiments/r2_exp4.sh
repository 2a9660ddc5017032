#!/bin/bash
# round 2 pass 4: no-speculation deref/compute occupancy variants, resident
# collage aligned + unaligned (two-phase straddle pins) vs round 1
mkdir -p gpurun_out
for v in vA vB vC; do
  AP_LIB_PATH=build/variants/lib_$v.so AP_DEREF_GRIDS=148,296,592 AP_FIG6_TBS=148,296 timeout 400 python tools/exp_hit.py
done > gpurun_out/r2_exp_hit4.txt 2>&1
for v in r1 vA; do
  for st in 4096 3072; do
    echo "== $v stride $st"; AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_STRIDE=$st AP_PROF_SCHEDS=2,1 timeout 600 python tools/prof_collage.py 1048576 4 8
  done
done > gpurun_out/r2_coll_res4.txt 2>&1
