#!/bin/bash
mkdir -p gpurun_out
s=$(date +%s)
python bench.py --steps 5 --warmup 3 > gpurun_out/r2_bench_default.json 2> gpurun_out/r2_bench_default.err
echo "rc=$? wall_s=$(( $(date +%s) - s ))" >> gpurun_out/r2_bench_default.err
