#!/bin/bash
mkdir -p gpurun_out /tmp/ncu
timeout 900 ncu --set full --import-source on --clock-control none -k regex:'^k_seq$' -s 3 -c 1 -o /tmp/ncu/r2_full_c1 -f \
  python bench.py --workload c1 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/r2_full_c1.out 2>&1
python tools/ncu_summary.py /tmp/ncu/r2_full_c1.ncu-rep 40 > gpurun_out/r2_full_c1.txt 2>&1
