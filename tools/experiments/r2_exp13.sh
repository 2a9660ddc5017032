#!/bin/bash
# round 2 pass 13: M2r ceiling microbenchmark, N>1 bench plumbing on one GPU,
# the hash-table ablation's parity suite (opt-in), C4 unaligned and C5 lines
mkdir -p gpurun_out
./tools/atomic_ceiling > gpurun_out/r2_atomic_ceiling.txt 2>&1
bash tools/validate_multirank.sh
AP_RUN_PT_HASH=1 timeout 900 python -m pytest tests/test_gpu_pt_hash.py -q -x > gpurun_out/r2_hash_tests.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_hash_tests.txt
timeout 900 python bench.py --workload c4 --stride 3072 --steps 3 --warmup 2 > gpurun_out/r2_bench_c4u.json 2> gpurun_out/r2_bench_c4u.err
timeout 1800 python bench.py --workload c5 --steps 3 --warmup 1 > gpurun_out/r2_bench_c5.json 2> gpurun_out/r2_bench_c5.err
echo "rc=$?" >> gpurun_out/r2_bench_c5.err
bash tools/fill_ncu.sh
bash tools/sanitize.sh
