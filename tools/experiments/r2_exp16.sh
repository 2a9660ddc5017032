#!/bin/bash
mkdir -p gpurun_out
bash tools/r2_hash.sh
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2_smoke.txt 2>&1
timeout 600 python tools/copy_bw.py > gpurun_out/r2_copy_bw.txt 2>&1
timeout 300 python tools/latency.py > gpurun_out/r2_latency.txt 2>&1
