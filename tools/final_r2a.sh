#!/bin/bash
# round-2 evidence refresh, part A: tests, smoke, bench lines, micro-suites,
# multirank plumbing (1 GPU).  Outputs under gpurun_out/final/.
mkdir -p gpurun_out/final
O=gpurun_out/final
timeout 1500 python -m pytest tests -m gpu -q > $O/gputest.txt 2>&1; tail -2 $O/gputest.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.txt 2>&1
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
timeout 900 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err
for w in c1 c3 c4 c5; do timeout 1200 python bench.py --workload $w > $O/bench_$w.json 2> $O/bench_$w.err; done
timeout 1200 python bench.py --workload c4 --stride 3072 > $O/bench_c4u.json 2> $O/bench_c4u.err
AP_DEREF_GRIDS=148,296,592 AP_FIG6_TBS=148,296 timeout 900 python tools/exp_hit.py > $O/exp_hit.txt 2>&1
timeout 600 python tools/copy_bw.py > $O/copy_bw.txt 2>&1
timeout 300 python tools/latency.py > $O/latency.txt 2>&1
AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 1 2 4 8 16 > $O/collage_resident.txt 2>&1
AP_PROF_STRIDE=3072 AP_PROF_SCHEDS=2 timeout 600 python tools/prof_collage.py 1048576 8 16 >> $O/collage_resident.txt 2>&1
bash tools/validate_multirank.sh
for f in gpurun_out/multirank_*; do mv $f $O/; done
echo done-a
