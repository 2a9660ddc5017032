#!/bin/bash
# ncu evidence for profiles/ (round 2): launch list of the default bench
# command, one --set full capture of each dominant kernel (apointer + raw twin
# where there is one), compute-sanitizer over the scenarios.  1 GPU.
# Reports stay in /tmp on the box; their text summaries come back.
mkdir -p gpurun_out /tmp/ncu
N="ncu --set full --import-source on --clock-control none"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file /tmp/ncu/r2_launches_c2.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline \
  > gpurun_out/r2_launches_c2.out 2>&1
python tools/launch_summary.py /tmp/ncu/r2_launches_c2.csv "ncu launch list of: python bench.py --steps 2 --warmup 1 --no-cpu-baseline" \
  > gpurun_out/r2_launches_c2_summary.txt 2>&1
gzip -c /tmp/ncu/r2_launches_c2.csv > gpurun_out/r2_launches_c2.csv.gz
timeout 900 $N -k regex:'^k_random$' -s 1 -c 1 -o /tmp/ncu/r2_full_c2 -f \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-collage > gpurun_out/r2_full_c2.out 2>&1
for k in k_seq k_seq_deref k_random; do
  timeout 900 $N -k regex:"^$k\$" -c 2 -o /tmp/ncu/r2_full_$k -f python tools/prof_kernels.py \
    > gpurun_out/r2_full_$k.out 2>&1
done
timeout 900 $N -k 'regex:^k_collage$' -s 1 -c 1 -o /tmp/ncu/r2_full_c4 -f \
  python bench.py --workload c4 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/r2_full_c4.out 2>&1
AP_PROF_SCHEDS=2 AP_PROF_STEPS=1 timeout 900 $N -k 'regex:^k_collage$' -s 1 -c 2 \
  -o /tmp/ncu/r2_full_c4_resident -f python tools/prof_collage.py 1048576 8 > gpurun_out/r2_full_c4_resident.out 2>&1
timeout 900 $N -k 'regex:^k_seq_queue$' -s 1 -c 1 -o /tmp/ncu/r2_full_c1 -f \
  python bench.py --workload c1 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/r2_full_c1.out 2>&1
for r in /tmp/ncu/*.ncu-rep; do
  b=$(basename $r .ncu-rep)
  python tools/ncu_summary.py $r 30 > gpurun_out/$b.txt 2>&1
done
echo ncu-done
bash tools/sanitize.sh
echo all-done
