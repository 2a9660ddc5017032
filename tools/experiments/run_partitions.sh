# GPU tests for the collage + both C5 partition projections + the N>1 bench plumbing (2 ranks sharing cuda:0)
timeout 900 python -m pytest tests/test_gpu_collage.py -x -q 2>&1 | tail -2
timeout 1200 python tools/c5_partitions.py 2 units > gpurun_out/c5_partitions_units.txt 2>&1; cat gpurun_out/c5_partitions_units.txt
timeout 1200 python tools/c5_partitions.py 2 blocks > gpurun_out/c5_partitions_blocks.txt 2>&1; cat gpurun_out/c5_partitions_blocks.txt
AP_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
    --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 1 --workload c4 \
    > gpurun_out/multirank_c4.json 2> gpurun_out/multirank_c4.err; echo "rc=$?"
python -c "import json;d=json.load(open('gpurun_out/multirank_c4.json'));print(d['value'], d['config']['parallelism'], d['collage'].get('gathered_parity_vs_oracle'), d['collage'].get('parity_vs_oracle'))"
