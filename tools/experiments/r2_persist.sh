# persistent pipelined collage (prod) vs per-item CTAs (ps0) vs persistent at 2 CTAs/SM (pm2)
mkdir -p gpurun_out/ps; O=gpurun_out/ps
timeout 900 python -m pytest tests/test_gpu_collage.py tests/test_gpu_mgpu.py -q -x > $O/tc.txt 2>&1; tail -2 $O/tc.txt
for v in prod ps0 pm2; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  echo "== $v" >> $O/res.txt
  AP_PROF_SCHEDS=2 timeout 300 python tools/prof_collage.py 1048576 4 8 16 >> $O/res.txt 2>&1
  AP_PROF_STRIDE=3072 AP_PROF_SCHEDS=2 timeout 300 python tools/prof_collage.py 1048576 8 >> $O/res.txt 2>&1
  timeout 600 python bench.py --workload c4 --no-cpu-baseline > $O/c4_$v.json 2>$O/c4_$v.err
  python -c "import json; d=json.load(open('$O/c4_$v.json')); print('$v cold c4', d['ms_per_step'], d.get('roofline',{}).get('frac'))" >> $O/res.txt 2>&1
done
cat $O/res.txt
