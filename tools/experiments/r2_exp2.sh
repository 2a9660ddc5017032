#!/bin/bash
# round 2, second GPU pass: new parity tests, per-access pipeline variants,
# resident collage (round-1 build vs the ABI-call build)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_reads.py tests/test_gpu_collage.py -m gpu -x -q > gpurun_out/r2_tests2.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_tests2.txt
for v in m1p6 m1p8 m1p12 m2p4; do
  AP_LIB_PATH=build/variants/lib_$v.so AP_DEREF_GRIDS=148,296,592 AP_FIG6_TBS=148,296 timeout 400 python tools/exp_hit.py
done > gpurun_out/r2_exp_hit2.txt 2>&1
for v in r1 p4; do
  echo "== $v"; AP_LIB_PATH=build/variants/lib_$v.so timeout 600 python tools/prof_collage.py 1048576 1 4 8
done > gpurun_out/r2_coll_res.txt 2>&1
