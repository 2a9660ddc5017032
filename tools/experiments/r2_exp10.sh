#!/bin/bash
# round 2 pass 10: GPU suite (drop-behind policy tests) + C1 / C3 lines
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2_tests10.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_tests10.txt
python bench.py --workload c1 --steps 5 --warmup 3 > gpurun_out/r2_bench_c1.json 2> gpurun_out/r2_bench_c1.err
python bench.py --workload c3 --steps 3 --warmup 2 > gpurun_out/r2_bench_c3.json 2> gpurun_out/r2_bench_c3.err
