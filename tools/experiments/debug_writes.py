import sys, time
import numpy as np, torch
sys.path.insert(0, "."); sys.path.insert(0, "tests")
import oracle, paper_conf_isca_shaharbs16_b200 as ap
from helpers import make_file
from oracle import invariants as inv
frames, grid, block, reads, policy = (int(x) for x in sys.argv[1:6])
mode = sys.argv[6] if len(sys.argv) > 6 else "w"
n = 2 << 20
f = make_file(n, seed=2)
want = oracle.apply_writes(f.copy(), 4, 1, nthreads=grid * block, reads=reads, seed=3)
c = ap.ap_cache_create(frames, 4096)
ap.ap_cache_set_tuning(c, 1, 64, 2000)
ap.ap_cache_set_policy(c, policy, 11)
r = ap.ap_mmap_prot(c, f, 3)
t = time.time()
if mode == "w":
    ap.ap_bench_write(c, r, ap.bench_cfg(ap.AP_UNIFORM, 4, grid, block, reads_per_thread=reads, seed=3))
else:
    out = torch.zeros(grid * block, dtype=torch.int64, device="cuda")
    ap.ap_bench_read(c, r, ap.bench_cfg(ap.AP_UNIFORM, 4, grid, block, reads_per_thread=reads, seed=3), out)
torch.cuda.synchronize()
print(mode, "kernel", round(time.time() - t, 3), "s err", ap.ap_last_device_error(c), ap.ap_cache_stats(c), flush=True)
pte = ap.ap_region_dump_pte(c, r)
st, ref, fr, rc = inv.pte_fields(pte)
dirty = (pte >> np.uint64(60)) & np.uint64(1)
for i in np.nonzero((st != 0) | (rc != 0))[0][:10]:
    print(f"  page {i}: state {st[i]} ref {ref[i]} dirty {int(dirty[i])} frame {fr[i]} rc {rc[i]}")
owner, left = ap.ap_cache_dump(c)
print("  owner", [hex(int(o)) for o in owner[:4]], "free_left", left)
