# C1: next work-queue unit taken after the current one (ql1) vs before (prod); 4 alternating rounds
mkdir -p gpurun_out/ql; O=gpurun_out/ql
for i in 1 2 3 4; do
for v in prod ql1; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  timeout 300 python bench.py --workload c1 --no-cpu-baseline --steps 10 > $O/c1_$v.json 2>$O/c1_$v.err
  python -c "import json; d=json.load(open('$O/c1_$v.json')); f=d['fault_bound']; print('$v c1', d['ms_per_step'], d['value'], f['frac_of_host_link'], 'waits', f['waits'], 'eq', f['raw_twin_equal'])" >> $O/res.txt
done
done
cat $O/res.txt
