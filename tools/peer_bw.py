"""N2 peer fills on one GPU: cache B (1 GiB) reads the C2 workload (4 GiB
file, 64 KiB pages, uniform-random 4-B reads, cold) with and without a peer
cache A on the same GPU that holds the whole file.  Prints B's fill rate
from each source.  Same-GPU peer copies are HBM-to-HBM; across GPUs the same
copies run over NVLink 5 (not measurable on a 1-GPU box)."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

GiB = 1 << 30
P = 65536
n = 4 * GiB
raw = np.empty(n + (1 << 21), np.uint8)
o = (-raw.ctypes.data) % (1 << 21)
f = synth.fill_file(raw[o:o + n], 1)
a = ap.ap_cache_create(n // P, P)
b = ap.ap_cache_create(GiB // P, P)
ra, rb = ap.ap_mmap(a, f), ap.ap_mmap(b, f)
ap.ap_prefill(a, ra, 0, n // P)
torch.cuda.synchronize()
grid, block = 148, 512
cfg = ap.bench_cfg(ap.AP_UNIFORM, 4, grid, block, reads_per_thread=8, seed=1234)
out = torch.empty(grid * block, dtype=torch.int64, device="cuda")
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
res = {}
for peer in (False, True, False, True):
    if peer:
        ap.ap_region_add_peer(b, rb, a, ra)
    ts, sts = [], []
    for i in range(4):
        ap.ap_cache_reset(b)
        s.record(); ap.ap_bench_read(b, rb, cfg, out); e.record(); e.synchronize()
        st = ap.ap_cache_stats(b)
        if i >= 1:
            ts.append(s.elapsed_time(e) * 1e-3); sts.append(st)
    ck = out.clone()
    t = float(np.mean(ts))
    st = sts[-1]
    moved = st["fill_bytes"] + st["peer_bytes"]
    print(f"peer={peer}: {t * 1e3:.1f} ms, majors {st['major']}, peer fills {st['peer_fills']}, "
          f"host fill {st['fill_bytes'] / t / 1e9:.1f} GB/s, peer fill {st['peer_bytes'] / t / 1e9:.1f} GB/s, "
          f"total {moved / t / 1e9:.1f} GB/s, err={ap.ap_last_device_error(b)}")
    res.setdefault(peer, ck)
    if peer:
        ap.ap_region_clear_peers(b, rb)
print("checksums equal with/without peer:", bool(torch.equal(res[False], res[True])))
