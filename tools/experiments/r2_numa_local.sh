# host files bound to the GPU's NUMA node (AP_NUMA_LOCAL=1, the bench default now) vs first-touch placement (0): C1 / C2 / C3 / C4, separate processes, alternating
mkdir -p gpurun_out/nl; O=gpurun_out/nl
cat /sys/devices/system/node/online > $O/res.txt; python -c "import torch,bench; print('gpu node', bench.gpu_numa_node(torch, torch.device('cuda:0')))" >> $O/res.txt 2>&1
for i in 1 2 3; do
for v in 1 0; do
  AP_NUMA_LOCAL=$v timeout 300 python bench.py --workload c1 --no-cpu-baseline > $O/c1.json 2>/dev/null
  python -c "import json; d=json.load(open('$O/c1.json')); print('local=$v c1', d['ms_per_step'], d['fault_bound']['frac_of_host_link'], d['step_times']['std_ms'] if 'step_times' in d else '')" >> $O/res.txt
done
done
for v in 1 0; do
  AP_NUMA_LOCAL=$v timeout 300 python bench.py --workload c3 --no-cpu-baseline > $O/c3.json 2>/dev/null
  python -c "import json; d=json.load(open('$O/c3.json')); print('local=$v c3', d['ms_per_step'], d['fault_bound']['frac_of_host_link'])" >> $O/res.txt
  AP_NUMA_LOCAL=$v timeout 300 python bench.py --workload c4 --no-cpu-baseline > $O/c4.json 2>/dev/null
  python -c "import json; d=json.load(open('$O/c4.json')); print('local=$v c4', d['ms_per_step'], d['roofline']['frac'])" >> $O/res.txt
  AP_NUMA_LOCAL=$v timeout 600 python bench.py --no-collage --no-reads --no-c5 --no-cpu-baseline > $O/c2.json 2>/dev/null
  python -c "import json; d=json.load(open('$O/c2.json')); print('local=$v c2', d['ms_per_step'], d['roofline']['frac'])" >> $O/res.txt
done
cat $O/res.txt
