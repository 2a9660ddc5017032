#!/bin/bash
# round 2 pass 12: what the resident collage's +28 % is made of: acquire link
# vs relaxed link, release unlink vs relaxed unlink (measurement-only builds)
mkdir -p gpurun_out
for v in s64 lr ur lur; do
  echo "== $v"
  AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 4 8
done > gpurun_out/r2_coll_order12.txt 2>&1
