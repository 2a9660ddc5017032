# precomputed window bounds + empty-window early exit: window sweep again, collage tests, resident check
mkdir -p gpurun_out/wb; O=gpurun_out/wb
timeout 900 python -m pytest tests/test_gpu_collage.py tests/test_gpu_mgpu.py -q -x > $O/tc.txt 2>&1; tail -1 $O/tc.txt >> $O/res.txt
for n in 12 32 64 128; do
  timeout 600 python bench.py --workload c4 --id-chunks $n --steps 3 $( [ $n = 32 ] || echo --no-cpu-baseline ) > $O/c4_$n.json 2>$O/c4_$n.err
  python -c "import json; d=json.load(open('$O/c4_$n.json')); c=d['collage']; print('c4 chunks $n', d['ms_per_step'], 'ms fills', c['fill_GB'], 'frac', d['roofline']['frac'], c.get('parity_vs_oracle'))" >> $O/res.txt 2>&1
done
for n in 12 16 24 32 48; do
  timeout 900 python bench.py --workload c5 --id-chunks $n --steps 3 $( [ $n = 24 ] || echo --no-cpu-baseline ) > $O/c5_$n.json 2>$O/c5_$n.err
  python -c "import json; d=json.load(open('$O/c5_$n.json')); c=d['collage']; print('c5 chunks $n', d['ms_per_step'], 'ms fills', c['fill_GB'], 'frac', d['roofline']['frac'], c.get('parity_vs_oracle'))" >> $O/res.txt 2>&1
done
AP_PROF_SCHEDS=2 timeout 300 python tools/prof_collage.py 1048576 8 >> $O/res.txt 2>&1
cat $O/res.txt
