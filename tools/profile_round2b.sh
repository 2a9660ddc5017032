#!/bin/bash
# round-2 final evidence (1 GPU): bench lines from the final code, the ncu
# launch list of the default bench command, --set full of the collage kernel
# (one fused-window launch = a whole cold C4 step) and of C1, sanitizer.
mkdir -p gpurun_out/final2 /tmp/ncu
O=gpurun_out/final2
timeout 1500 python -m pytest tests -m gpu -q > $O/gputest.txt 2>&1; tail -1 $O/gputest.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.txt 2>&1
timeout 1200 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
timeout 600 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err
for w in c1 c3 c4 c5; do timeout 1200 python bench.py --workload $w > $O/bench_$w.json 2> $O/bench_$w.err; done
timeout 1200 python bench.py --workload c4 --stride 3072 > $O/bench_c4u.json 2> $O/bench_c4u.err
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file /tmp/ncu/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > $O/launches.out 2>&1
python tools/launch_summary.py /tmp/ncu/launches.csv "ncu launch list of: python bench.py --steps 2 --warmup 1 --no-cpu-baseline" > $O/launches_summary.txt 2>&1
gzip -c /tmp/ncu/launches.csv > $O/launches.csv.gz
N="ncu --set full --import-source on --clock-control none"
timeout 900 $N -k 'regex:^k_collage$' -s 1 -c 1 -o /tmp/ncu/full_c4 -f \
  python bench.py --workload c4 --steps 1 --warmup 1 --no-cpu-baseline > $O/full_c4.out 2>&1
AP_PROF_SCHEDS=2 AP_PROF_STEPS=1 timeout 900 $N -k 'regex:^k_collage$' -s 1 -c 2 \
  -o /tmp/ncu/full_c4_resident -f python tools/prof_collage.py 1048576 8 > $O/full_c4_resident.out 2>&1
timeout 900 $N -k 'regex:^k_random$' -s 1 -c 1 -o /tmp/ncu/full_c2 -f \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-collage --no-reads > $O/full_c2.out 2>&1
for r in /tmp/ncu/*.ncu-rep; do
  b=$(basename $r .ncu-rep)
  python tools/ncu_summary.py $r 30 > $O/$b.txt 2>&1
done
bash tools/sanitize.sh; mv gpurun_out/sanitize.txt $O/sanitize.txt
echo all-done
