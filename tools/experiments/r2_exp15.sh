#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2_tests15.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_tests15.txt
bash tools/r2_hash.sh
AP_RUN_PT_HASH=1 timeout 900 python -m pytest tests/test_gpu_pt_hash.py -q -rxX > gpurun_out/r2_hash_tests.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_hash_tests.txt
