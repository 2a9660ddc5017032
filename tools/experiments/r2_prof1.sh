#!/bin/bash
# ncu --set full of the per-access dereference (apointer + raw twin)
mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:k_seq_deref --launch-skip 2 -c 2 \
    -o gpurun_out/deref_m2p4 -f python tools/prof_deref.py > gpurun_out/deref_m2p4.log 2>&1
echo "rc=$?" >> gpurun_out/deref_m2p4.log
