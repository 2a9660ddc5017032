#!/bin/bash
# per-access deref / Fig. 6 after the C1 fault-path changes: pre (before them), lean (miss path without
# the pin / claim-first probe), leannolm (lean without the link_minor pool/stats hoist)
mkdir -p gpurun_out
( for v in pre lean leannolm pre lean leannolm; do
  echo "== $v"; AP_LIB_PATH=build/variants/lib_$v.so AP_DEREF_GRIDS=148 AP_FIG6_TBS=148 timeout 400 python tools/exp_hit.py | grep -E "deref|read|add|reduce"
done ) > gpurun_out/r2_lean.txt 2>&1
