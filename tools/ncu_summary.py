"""Summarise an ncu report: key metrics + top stall PCs (for profiles/)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
topn = int(sys.argv[2]) if len(sys.argv) > 2 else 25


def ncu(*a):
    return subprocess.run(["ncu", "-i", rep, *a], capture_output=True, text=True).stdout


rows = list(csv.reader(io.StringIO(ncu("--page", "details", "--csv"))))
hdr = rows[0]
ki, mi, vi, ui = (hdr.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
want = ["Duration", "DRAM Throughput", "Memory Throughput", "Executed Ipc Active", "Issue Slots Busy",
        "Achieved Occupancy", "Registers Per Thread", "Executed Instructions",
        "Warp Cycles Per Issued Instruction", "Eligible Warps Per Scheduler", "L2 Hit Rate",
        "SM Frequency", "DRAM Frequency"]
seen = set()
for r in rows[1:]:
    if r[mi] in want and (r[ki], r[mi]) not in seen:
        seen.add((r[ki], r[mi]))
        print(f"{r[ki][:60]} | {r[mi]} = {r[vi]} {r[ui]}")
raw = list(csv.reader(io.StringIO(ncu("--page", "raw", "--csv"))))
for rr in raw[2:]:
    d = dict(zip(raw[0], rr))
    for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum",
              "smsp__inst_executed.sum", "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum"):
        if k in d:
            print(f"raw {k} = {d[k]} {dict(zip(raw[0], raw[1])).get(k, '')}")
    # local-memory (spill) traffic, whatever this ncu version calls it
    for k in sorted(d):
        if "local" in k and k.endswith(".sum") and ("inst" in k or "bytes" in k or "sectors" in k):
            print(f"raw {k} = {d[k]} {dict(zip(raw[0], raw[1])).get(k, '')}")
    st = sorted(((float(v.replace(",", "")), k) for k, v in d.items()
                 if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")
                 and v.replace(",", "").replace(".", "").isdigit()), reverse=True)[:8]
    print("stalls:", ", ".join(f"{k.split('stalled_')[1]}={int(v)}" for v, k in st))
src = list(csv.reader(io.StringIO(ncu("--page", "source", "--csv", "--print-source", "sass"))))
h = src[1]
i_src, i_s, i_e = h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
data = [r for r in src[2:] if len(r) == len(h) and r[i_s].isdigit()]
tot = sum(int(r[i_s]) for r in data) or 1
print(f"top stall PCs (of {tot} samples):")
for r in sorted(data, key=lambda r: -int(r[i_s]))[:topn]:
    print(f"  {r[0][-5:]} {int(r[i_s]) * 100 / tot:5.1f}% exec={r[i_e]:>8} {r[i_src].strip()[:70]}")
