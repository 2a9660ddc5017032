mkdir -p gpurun_out/wc; O=gpurun_out/wc
timeout 1500 python -m pytest tests -m gpu -q -x > $O/gputest.txt 2>&1; tail -1 $O/gputest.txt
timeout 900 python bench.py --workload c5 > $O/c5.json 2>$O/c5.err
timeout 900 python bench.py --workload c4 > $O/c4.json 2>$O/c4.err
for w in c4 c5; do python -c "import json; d=json.load(open('$O/$w.json')); c=d['collage']; print('$w', d['ms_per_step'], 'ms fills', c['fill_GB'], 'frac', d['roofline']['frac'], c.get('parity_vs_oracle'), d.get('cpu_baseline'))"; done
bash tools/validate_multirank.sh; for f in gpurun_out/multirank_*.err; do echo "$f $(tail -1 $f)"; done
