#!/bin/bash
# One-off probe of the GPU box: host cores, RAM, NUMA, PCIe, shm, H2D bandwidth.
mkdir -p gpurun_out
{
echo "== nproc"; nproc
echo "== lscpu"; lscpu | head -30
echo "== free"; free -g
echo "== shm"; df -h /dev/shm
echo "== numa"; ls /sys/devices/system/node/ | grep node; cat /sys/devices/system/node/node*/meminfo 2>/dev/null | grep MemTotal
echo "== nvidia-smi"; nvidia-smi; nvidia-smi topo -m
echo "== pcie"; nvidia-smi --query-gpu=index,pcie.link.gen.current,pcie.link.gen.max,pcie.link.width.current,pcie.link.width.max --format=csv
echo "== ulimit"; ulimit -a
python - <<'PY'
import torch, time
print(torch.cuda.get_device_properties(0))
for sz in [256<<20, 1<<30]:
    h = torch.empty(sz, dtype=torch.uint8, pin_memory=True); d = torch.empty(sz, dtype=torch.uint8, device='cuda')
    for _ in range(3): d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    s=torch.cuda.Event(enable_timing=True); e=torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(10): d.copy_(h, non_blocking=True)
    e.record(); torch.cuda.synchronize()
    print("H2D pinned", sz, 10*sz/(s.elapsed_time(e)/1e3)/1e9, "GB/s")
    s.record()
    for _ in range(10): h.copy_(d, non_blocking=True)
    e.record(); torch.cuda.synchronize()
    print("D2H pinned", sz, 10*sz/(s.elapsed_time(e)/1e3)/1e9, "GB/s")
PY
} > gpurun_out/probe.txt 2>&1
