#!/bin/bash
# ncu evidence for profiles/: launch list of the default bench command, and
# one --set full capture of each dominant kernel.  Run under gpurun (1 GPU).
set -x
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_c2.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline \
  > gpurun_out/launches_c2.out 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_random -s 1 -c 1 \
  -o gpurun_out/full_c2 python bench.py --steps 1 --warmup 1 --no-cpu-baseline \
  > gpurun_out/full_c2.out 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_seq -c 1 \
  -o gpurun_out/full_hit python tools/prof_hit.py 65536 2 > gpurun_out/full_hit.out 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_seq -s 6 -c 1 \
  -o gpurun_out/full_hit_raw python tools/prof_hit.py 65536 2 > gpurun_out/full_hit_raw.out 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k 'regex:^k_collage$' -s 1 -c 1 \
  -o gpurun_out/full_c4 python bench.py --workload c4 --steps 1 --warmup 1 --no-cpu-baseline \
  > gpurun_out/full_c4.out 2>&1
AP_PROF_STEPS=1 timeout 900 ncu --set full --import-source on --clock-control none -k 'regex:^k_collage$' -c 2 \
  -o gpurun_out/full_c4_resident python tools/prof_collage.py 1048576 8 > gpurun_out/full_c4_resident.out 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_random -c 2 \
  -o gpurun_out/full_minor python tools/prof_minor.py > gpurun_out/full_minor.out 2>&1
echo done
# bench lines (outside ncu): default C2, C1, C3, C4, C4 unaligned, C5 (1 GPU)
timeout 600 python bench.py > gpurun_out/final_c2.json 2> gpurun_out/final_c2.err
for w in c1 c3 c4; do timeout 900 python bench.py --workload $w > gpurun_out/final_$w.json 2> gpurun_out/final_$w.err; done
timeout 900 python bench.py --workload c4 --stride 3072 > gpurun_out/final_c4u.json 2> gpurun_out/final_c4u.err
timeout 1500 python bench.py --workload c5 --steps 3 --warmup 1 > gpurun_out/final_c5.json 2> gpurun_out/final_c5.err
timeout 300 python bench.py --impl reference > gpurun_out/final_ref.json 2> gpurun_out/final_ref.err
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.txt 2>&1
timeout 600 python tools/fig6_sweep.py > gpurun_out/final_fig6.txt 2>&1
timeout 300 python tools/latency.py > gpurun_out/final_latency.txt 2>&1
echo bench-done
timeout 300 python tools/peer_bw.py > gpurun_out/final_peer_bw.txt 2>&1
for k in 12 16; do timeout 600 python bench.py --workload c4 --id-chunks $k --no-cpu-baseline > gpurun_out/final_c4_win$k.json 2>/dev/null; done
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/final_gpu_tests.txt 2>&1
echo all-done
