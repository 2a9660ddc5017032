#!/bin/bash
mkdir -p gpurun_out
( for b in 64,4096 64,16384 256,65536 1024,16384; do for sw in 64 4; do
  echo "== backoff $b sweep $sw"; AP_EXP_BACKOFF=$b AP_EXP_SWEEP=$sw AP_EXP_PATTERN=3 AP_EXP_FRAMES=64,64 AP_EXP_GRIDS=148 timeout 300 python tools/exp_c1.py
done; done ) > gpurun_out/r2_backoff.txt 2>&1
