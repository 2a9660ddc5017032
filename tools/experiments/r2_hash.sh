#!/bin/bash
# the hash-table page table (N4 ablation): which parity cases fail, and how
mkdir -p gpurun_out
AP_LIB_PATH=paper_conf_isca_shaharbs16_b200/libapointer_hash.so timeout 600 python -m pytest \
  tests/test_gpu_reads.py tests/test_gpu_collage.py -q -p no:cacheprovider --timeout 60 -x \
  > gpurun_out/r2_hash_detail.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_hash_detail.txt
