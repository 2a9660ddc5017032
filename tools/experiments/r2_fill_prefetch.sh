# fill prefetch (host reads of a claimed page issued before the frame allocation) vs without (fp0)
mkdir -p gpurun_out/fp; O=gpurun_out/fp
timeout 1500 python -m pytest tests -m gpu -q -x > $O/gputest.txt 2>&1; tail -1 $O/gputest.txt >> $O/res.txt
for i in 1 2; do
for v in prod fp0; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  for w in c1 c3 c4; do
    timeout 600 python bench.py --workload $w --no-cpu-baseline > $O/${w}_$v.json 2>$O/${w}_$v.err
    python -c "import json; d=json.load(open('$O/${w}_$v.json')); print('$v $w', d['ms_per_step'], 'ms', d['value'], d.get('roofline',{}).get('frac'))" >> $O/res.txt 2>&1
  done
  timeout 600 python bench.py --no-collage --no-reads --no-cpu-baseline > $O/c2_$v.json 2>$O/c2_$v.err
  python -c "import json; d=json.load(open('$O/c2_$v.json')); print('$v c2', d['ms_per_step'], 'ms fills', d['roofline']['achieved'], d['roofline']['frac'], 'hit', d['hit']['overhead_vs_raw'], 'deref', d['hit']['deref_vs_raw_per_access_twin']['overhead'], 'minor', d['minor']['frac_of_ceiling'])" >> $O/res.txt 2>&1
done
done
cat $O/res.txt
