mkdir -p gpurun_out/w1; O=gpurun_out/w1
timeout 900 python -m pytest tests/test_gpu_collage.py -q -x > $O/tc.txt 2>&1; tail -2 $O/tc.txt
for v in prod wide0; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  echo "== $v" >> $O/res.txt
  AP_PROF_SCHEDS=2 timeout 300 python tools/prof_collage.py 1048576 4 8 16 >> $O/res.txt 2>&1
  AP_PROF_STRIDE=3072 AP_PROF_SCHEDS=2 timeout 300 python tools/prof_collage.py 1048576 4 8 16 >> $O/res.txt 2>&1
done
unset AP_LIB_PATH
timeout 600 python bench.py --workload c4 > $O/c4.json 2>$O/c4.err
cat $O/res.txt; python -c "import json;d=json.load(open('$O/c4.json'));print(d['value'],d.get('ms_per_step'), {k:v for k,v in d.items() if k in ('resident','parity_vs_oracle')})"
