#!/bin/bash
# link_minor: pool/stats read before the acquire (lmhoist) vs HEAD (base), and the relaxed-link ablation
mkdir -p gpurun_out
for v in base lmhoist relaxed lmrelaxed; do
  echo "== $v"; AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 4 8 | grep N=
  AP_LIB_PATH=build/variants/lib_$v.so AP_PROF_STRIDE=3072 AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 8 | grep N=
  AP_LIB_PATH=build/variants/lib_$v.so timeout 300 python tools/prof_minor.py 2>&1 | tail -2
done > gpurun_out/r2_lm.txt 2>&1
