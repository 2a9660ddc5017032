"""profiles/traffic.json from the ncu --set full summaries in profiles/ (DRAM
read + write bytes per launch of each dominant kernel)."""
import json
import re


def first_bytes(path, idx=0):
    t = open(path).read()
    rd = re.findall(r'raw dram__bytes_read.sum = ([0-9.]+) (\w+)', t)
    wr = re.findall(r'raw dram__bytes_write.sum = ([0-9.]+) (\w+)', t)
    mul = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}
    return float(rd[idx][0]) * mul[rd[idx][1]] + float(wr[idx][0]) * mul[wr[idx][1]]


tj = {
    "k_random<uint32_t, UNIFORM, apointer>": {"dram_bytes_per_launch": first_bytes('profiles/r01_full_c2.txt'), "source": "profiles/r01_full_c2.txt (ncu --set full, 1 launch; DRAM read + write: the frame fills are the writes)"},
    "k_seq<uint4, apointer>": {"dram_bytes_per_launch": first_bytes('profiles/r01_full_hit.txt'), "source": "profiles/r01_full_hit.txt (ncu --set full, 1 launch, 2 passes over 1 GiB)"},
    "k_seq<uint4, raw>": {"dram_bytes_per_launch": first_bytes('profiles/r01_full_hit_raw.txt'), "source": "profiles/r01_full_hit_raw.txt (ncu --set full, 1 launch, 2 passes over 1 GiB)"},
    "k_collage<8, apointer>": {"dram_bytes_per_launch": first_bytes('profiles/r01_full_c4.txt'), "source": "profiles/r01_full_c4.txt (ncu --set full, 1 launch = one of the 12 record-id window passes of a cold C4 step)"},
    "k_collage<8, apointer> resident": {"dram_bytes_per_launch": first_bytes('profiles/r01_full_c4_resident.txt', 1), "source": "profiles/r01_full_c4_resident.txt (second kernel: the resident-cache run; the first is the cold run that fills the cache)"},
    "k_random<uint32_t, UNIFORM, apointer> resident (M2r)": {"dram_bytes_per_launch": first_bytes('profiles/r01_full_minor.txt'), "source": "profiles/r01_full_minor.txt (ncu --set full; first launch = apointer, second = raw twin)"},
}
json.dump(tj, open('profiles/traffic.json', 'w'), indent=1)
print(json.dumps({k: v["dram_bytes_per_launch"] for k, v in tj.items()}, indent=1))
