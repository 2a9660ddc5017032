# fused window passes with one warp per (window, unit) item (prod) vs one CTA per item (wu0)
mkdir -p gpurun_out/wu; O=gpurun_out/wu
timeout 900 python -m pytest tests/test_gpu_collage.py tests/test_gpu_mgpu.py -q -x > $O/tc.txt 2>&1; tail -1 $O/tc.txt >> $O/res.txt
for v in prod wu0; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  for n in 12 32 64; do
    timeout 600 python bench.py --workload c4 --id-chunks $n --steps 3 $( [ $n = 32 ] || echo --no-cpu-baseline ) > $O/c4_${v}_$n.json 2>$O/c4_${v}_$n.err
    python -c "import json; d=json.load(open('$O/c4_${v}_$n.json')); c=d['collage']; print('$v c4 chunks $n', d['ms_per_step'], 'ms fills', c['fill_GB'], 'frac', d['roofline']['frac'], c.get('parity_vs_oracle'))" >> $O/res.txt 2>&1
  done
  for n in 12 24 48 96; do
    timeout 900 python bench.py --workload c5 --id-chunks $n --steps 3 $( [ $n = 48 ] || echo --no-cpu-baseline ) > $O/c5_${v}_$n.json 2>$O/c5_${v}_$n.err
    python -c "import json; d=json.load(open('$O/c5_${v}_$n.json')); c=d['collage']; print('$v c5 chunks $n', d['ms_per_step'], 'ms fills', c['fill_GB'], 'frac', d['roofline']['frac'], c.get('parity_vs_oracle'))" >> $O/res.txt 2>&1
  done
done
cat $O/res.txt
