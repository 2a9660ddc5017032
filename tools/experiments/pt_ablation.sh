# N4 ablation: dense PTE array (libapointer.so) vs the paper's hash-table page table
# (libapointer_hash.so): hit mode, M2r minor faults, C2 fault-bound, resident collage
for i in 1 2; do for v in dense hash; do
  if [ $v = dense ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=paper_conf_isca_shaharbs16_b200/libapointer_hash.so; fi
  echo "== $v round $i"
  AP_LIB_PATH=$L timeout 300 python tools/prof_hit.py 65536 8 | grep -E "tile|range"
  AP_LIB_PATH=$L timeout 300 python tools/prof_minor.py 2>&1 | tail -1
  AP_LIB_PATH=$L timeout 300 python tools/prof_collage.py 1048576 8 2>&1 | grep sched=1
  AP_LIB_PATH=$L timeout 600 python bench.py --no-cpu-baseline --steps 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('C2 fill GB/s', d['value'], 'frac', d['roofline']['frac'])"
done; done
