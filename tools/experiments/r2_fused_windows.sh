# fused record-id windows (one launch per collage step) vs one launch per window (AP_COLLAGE_FUSED_WINDOWS=0)
mkdir -p gpurun_out/fw; O=gpurun_out/fw
timeout 900 python -m pytest tests/test_gpu_collage.py tests/test_gpu_mgpu.py -q -x > $O/tc.txt 2>&1; tail -2 $O/tc.txt
for i in 1 2; do
for v in prod fw0; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  timeout 600 python bench.py --workload c4 --no-cpu-baseline > $O/c4_$v.json 2>$O/c4_$v.err
  timeout 600 python bench.py --workload c4 --stride 3072 --no-cpu-baseline > $O/c4u_$v.json 2>$O/c4u_$v.err
  python - <<PY >> $O/res.txt
import json
for n in ("c4", "c4u"):
    d = json.load(open("$O/%s_$v.json" % n))
    print("$v", n, d["ms_per_step"], "ms", d.get("roofline", {}).get("frac"), d.get("parity_vs_oracle"))
PY
done
done
unset AP_LIB_PATH
for v in prod fw0; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  timeout 900 python bench.py --workload c5 --steps 3 --warmup 3 --no-cpu-baseline > $O/c5_$v.json 2>$O/c5_$v.err
  python -c "import json; d=json.load(open('$O/c5_$v.json')); print('$v c5', d['ms_per_step'], d.get('roofline',{}).get('frac'))" >> $O/res.txt
done
unset AP_LIB_PATH
/usr/bin/time -f "default bench wall %e s" timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; tail -1 $O/bench.err >> $O/res.txt
cat $O/res.txt
