#!/bin/bash
# round-2 final evidence after the collage window work (1 GPU): bench lines,
# launch list of the default command, --set full of C4 (CTA items) and C5
# (warp items) steps, GPU tests, smoke.
mkdir -p gpurun_out/final3 /tmp/ncu
O=gpurun_out/final3
timeout 1500 python -m pytest tests -m gpu -q > $O/gputest.txt 2>&1; tail -1 $O/gputest.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.txt 2>&1
timeout 1200 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
timeout 600 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err
for w in c1 c3 c4 c5; do timeout 1200 python bench.py --workload $w > $O/bench_$w.json 2> $O/bench_$w.err; done
timeout 1200 python bench.py --workload c4 --stride 3072 > $O/bench_c4u.json 2> $O/bench_c4u.err
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file /tmp/ncu/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > $O/launches.out 2>&1
python tools/launch_summary.py /tmp/ncu/launches.csv "ncu launch list of: python bench.py --steps 2 --warmup 1 --no-cpu-baseline" > $O/launches_summary.txt 2>&1
gzip -c /tmp/ncu/launches.csv > $O/launches.csv.gz
N="ncu --set full --import-source on --clock-control none"
timeout 900 $N -k 'regex:^k_collage$' -s 1 -c 1 -o /tmp/ncu/full_c4 -f \
  python bench.py --workload c4 --steps 1 --warmup 1 --no-cpu-baseline > $O/full_c4.out 2>&1
timeout 1500 $N -k 'regex:^k_collage_wunit$' -s 1 -c 1 -o /tmp/ncu/full_c5 -f \
  python bench.py --workload c5 --steps 1 --warmup 1 --no-cpu-baseline > $O/full_c5.out 2>&1
for r in /tmp/ncu/*.ncu-rep; do
  b=$(basename $r .ncu-rep)
  python tools/ncu_summary.py $r 30 > $O/$b.txt 2>&1
done
echo all-done
