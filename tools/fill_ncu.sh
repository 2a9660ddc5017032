#!/bin/bash
# ncu counters behind the fill A/B (S8): warp zero-copy LDG vs TMA bulk
# copies, host -> HBM; summaries of the sysmem / PCIe / DRAM metrics.
mkdir -p gpurun_out /tmp/ncu
ncu --query-metrics 2>/dev/null | grep -i -E "pcie|sysmem|nvlink|c2c" > gpurun_out/r2_ncu_sysmem_metrics.txt
for k in k_ldg k_tma; do
  timeout 600 ncu --set full --clock-control none -k regex:"^$k\$" -c 1 -o /tmp/ncu/r2_fill_$k -f ./tools/fill_mb \
    > gpurun_out/r2_fill_$k.out 2>&1
  ncu -i /tmp/ncu/r2_fill_$k.ncu-rep --page raw --csv > /tmp/ncu/r2_fill_$k.csv 2>&1
  python - "$k" <<'PY' > gpurun_out/r2_fill_$k.txt
import csv, sys
rows = list(csv.reader(open(f"/tmp/ncu/r2_fill_{sys.argv[1]}.csv")))
h, u, v = rows[0], rows[1], rows[2]
for name, unit, val in zip(h, u, v):
    n = name.lower()
    if any(s in n for s in ("sysmem", "pcie", "dram__bytes", "gpu__time_duration", "dram__throughput",
                            "lts__t_sectors_aperture", "l1tex__m_xbar2l1tex", "smsp__inst_executed.sum",
                            "sm__throughput.avg.pct", "launch__grid_size", "launch__block_size")):
        print(f"{name} = {val} {unit}")
PY
done
