# record-id window count (id_chunks) with fused windows: C4 and C5 cold steps
mkdir -p gpurun_out/ws; O=gpurun_out/ws
for n in 8 12 16 24 32; do
  timeout 600 python bench.py --workload c4 --id-chunks $n --no-cpu-baseline --steps 3 > $O/c4_$n.json 2>$O/c4_$n.err
  python -c "import json; d=json.load(open('$O/c4_$n.json')); c=d['collage']; print('c4 chunks $n', d['ms_per_step'], 'ms fills', c['fill_GB'], 'frac', d['roofline']['frac'])" >> $O/res.txt 2>&1
done
for n in 8 12 16 24; do
  timeout 900 python bench.py --workload c5 --id-chunks $n --no-cpu-baseline --steps 3 > $O/c5_$n.json 2>$O/c5_$n.err
  python -c "import json; d=json.load(open('$O/c5_$n.json')); c=d['collage']; print('c5 chunks $n', d['ms_per_step'], 'ms fills', c['fill_GB'], 'frac', d['roofline']['frac'])" >> $O/res.txt 2>&1
done
AP_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 1 --workload c4 > $O/mr_c4.json 2> $O/mr_c4.err
python -c "
import json; d=json.loads(open('$O/mr_c4.json').read().strip().splitlines()[-1]); c=d['collage']; print('mr c4 raw_twin_equal', c['raw_twin_equal'], {k:v.get('equal') for k,v in c['resident_cache'].items() if isinstance(v,dict)}, c['gathered_parity_vs_oracle'])" >> $O/res.txt 2>&1
cat $O/res.txt
