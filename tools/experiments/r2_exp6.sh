#!/bin/bash
# round 2 pass 6: the new default bench line end to end (C2 + hit + minor +
# embedded C4 collage), the reference arm, and an ncu capture of the resident
# collage (apointer + raw twin)
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2_smi6.txt 2>&1
/usr/bin/time -v python bench.py --steps 5 --warmup 3 > gpurun_out/r2_bench_default.json 2> gpurun_out/r2_bench_default.err
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r2_bench_ref.json 2> gpurun_out/r2_bench_ref.err
AP_PROF_SCHEDS=2 AP_PROF_STEPS=1 ncu --set full --import-source on --clock-control none -k regex:k_collage \
  --launch-skip 1 -c 2 -o gpurun_out/coll_res_g8 -f python tools/prof_collage.py 1048576 8 > gpurun_out/coll_res_g8.log 2>&1
