#!/bin/bash
# Exercise bench.py's N>1 paths on a single GPU (both ranks on cuda:0, gloo
# collectives).  Correctness/plumbing check only -- not bench numbers.
mkdir -p gpurun_out
run() {
  name=$1; shift
  AP_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
    --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 1 "$@" \
    > gpurun_out/multirank_$name.json 2> gpurun_out/multirank_$name.err
  echo "rc=$?" >> gpurun_out/multirank_$name.err
}
run c2_default
run c4_fused --workload c4
run c4_nccl --workload c4 --combine nccl
run c4_blocks_fused --workload c4 --partition blocks
