"""profiles/traffic.json from the ncu --set full summaries in profiles/ (DRAM
read + write bytes per launch of each dominant kernel; every summary names
its kernels in capture order: apointer first, then the raw twin)."""
import json
import re
import sys

R = sys.argv[1] if len(sys.argv) > 1 else "r02"


def kernel_bytes(path):
    """[(kernel line, dram read + write bytes)] in the order of the report."""
    t = open(path).read()
    names = [m for m in re.findall(r"^(.*?) \| Duration", t, re.M)]
    rd = re.findall(r'raw dram__bytes_read.sum = ([0-9.]+) (\w+)', t)
    wr = re.findall(r'raw dram__bytes_write.sum = ([0-9.]+) (\w+)', t)
    mul = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}
    return [(n, float(a[0]) * mul[a[1]] + float(b[0]) * mul[b[1]]) for n, a, b in zip(names, rd, wr)]


def entry(path, idx, what):
    ks = kernel_bytes(path)
    name, b = ks[idx]
    return {"dram_bytes_per_launch": b, "kernel_in_capture": name.strip(),
            "source": f"{path} (ncu --set full; {what})"}


tj = {
    "k_random<uint32_t, UNIFORM, apointer>": entry(f"profiles/{R}_full_c2.txt", 0, "one C2 launch, cold cache: the frame fills are the writes"),
    "k_seq<uint4, apointer>": entry(f"profiles/{R}_full_k_seq.txt", 0, "tile hit mode, 2 passes over 1 GiB"),
    "k_seq<uint4, raw>": entry(f"profiles/{R}_full_k_seq.txt", 1, "raw twin of the same launch"),
    "k_seq_deref<uint4, apointer>": entry(f"profiles/{R}_full_k_seq_deref.txt", 0, "per-access form, 2 passes over 1 GiB"),
    "k_seq_deref<uint4, raw>": entry(f"profiles/{R}_full_k_seq_deref.txt", 1, "raw twin of the same launch"),
    "k_random<uint32_t, UNIFORM, apointer> resident (M2r)": entry(f"profiles/{R}_full_k_random.txt", 0, "M2r: uniform 4-B reads over the resident GiB"),
    "k_random<uint32_t, UNIFORM, raw> resident (M2r)": entry(f"profiles/{R}_full_k_random.txt", 1, "the raw gather twin"),
    "k_collage<8, apointer>": entry(f"profiles/{R}_full_c4.txt", 0, "one launch = a whole cold C4 step (the 12 record-id window passes fused into one launch)"),
    "k_seq_queue<uint4, apointer>": entry(f"profiles/{R}_full_c1.txt", 0, "one C1 step: the 16 MiB file and its 64 frames live in L2, so DRAM sees almost nothing"),
    "k_random<uint32_t, DIVERGENT, apointer>": entry(f"profiles/{R}_full_c3.txt", 0, "one C3 step, cold 256 MiB cache: fills recycle frames whose dirty lines L2 absorbs, so DRAM writes are below the fill bytes"),
    "k_collage_wunit<8, apointer>": entry(f"profiles/{R}_full_c5.txt", 0, "one launch = a whole cold C5 step (96 record-id windows, one warp per (window, unit) item)"),
    "k_collage<8, apointer> resident": entry(f"profiles/{R}_full_c4_resident.txt", 0, "cache holds every record"),
    "k_collage<8, raw> resident": entry(f"profiles/{R}_full_c4_resident.txt", 1, "raw twin on an HBM copy"),
}
json.dump(tj, open('profiles/traffic.json', 'w'), indent=1)
print(json.dumps({k: (v["dram_bytes_per_launch"], v["kernel_in_capture"][:50]) for k, v in tj.items()}, indent=1))
