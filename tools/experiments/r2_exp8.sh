#!/bin/bash
# round 2 pass 8: resident collage groups 8/16/32 aligned + unaligned; ncu of
# the resident apointer collage and its raw twin (group 8)
mkdir -p gpurun_out
for st in 4096 3072; do
  echo "== stride $st"; AP_PROF_STRIDE=$st AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 8 16 32
done > gpurun_out/r2_coll_res8.txt 2>&1
AP_PROF_SCHEDS=2 AP_PROF_STEPS=1 ncu --set full --import-source on --clock-control none -k regex:'^k_collage$' \
  --launch-skip 1 -c 2 -o gpurun_out/coll_res_g8 -f python tools/prof_collage.py 1048576 8 > gpurun_out/coll_res_g8.log 2>&1
