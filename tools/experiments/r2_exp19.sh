#!/bin/bash
mkdir -p gpurun_out
for v in base idpf base idpf; do
  echo "== $v"; AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 8
  AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_STRIDE=3072 AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 8 | grep N=
done > gpurun_out/r2_idpf19.txt 2>&1
