# sweep quiet period (AP_SWEEP_QUIET) A/B on C1 + full GPU suite + default bench wall time
mkdir -p gpurun_out/q; O=gpurun_out/q
timeout 1500 python -m pytest tests -m gpu -q -x > $O/gputest.txt 2>&1; tail -2 $O/gputest.txt
P=$(python -c "import paper_conf_isca_shaharbs16_b200 as ap; print(ap.AP_SEQ_QUEUE)")
for i in 1 2; do
for v in prod q0; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  timeout 300 python bench.py --workload c1 --no-cpu-baseline > $O/c1_$v.json 2>$O/c1_$v.err
  python -c "import json; d=json.load(open('$O/c1_$v.json')); f=d['fault_bound']; print('$v c1', d['ms_per_step'], d['value'], f['frac_of_host_link'], 'waits', f['waits'], 'eq', f['raw_twin_equal'], f['other_policies'])" >> $O/res.txt
  AP_EXP_PATTERN=$P AP_EXP_FRAMES=64,96 AP_EXP_GRIDS=64,148 timeout 120 python tools/exp_c1.py | sed "s/^/$v /" >> $O/res.txt 2>&1
done
done
unset AP_LIB_PATH
t0=$(date +%s); timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; t1=$(date +%s); echo "default bench wall $((t1-t0)) s" >> $O/res.txt
cat $O/res.txt
