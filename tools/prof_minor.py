"""M2r: uniform-random 4-B apointer reads over a resident GiB --
every read is an unlink + a minor fault -- vs the raw gather from an HBM copy.
Prints CUDA-event timings; run under ncu for counters (-k regex:k_random).
Env: AP_LIB_PATH (library variant), AP_GRID (default 592), AP_READS (8)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

GiB = 1 << 30
page = 65536
grid, block = int(os.environ.get("AP_GRID", 592)), 512
reads = int(os.environ.get("AP_READS", 8))
raw = np.empty(GiB + (1 << 21), np.uint8)
o = (-raw.ctypes.data) % (1 << 21)
f = synth.fill_file(raw[o:o + GiB], 1)
c = ap.ap_cache_create(GiB // page, page)
r = ap.ap_mmap(c, f)
ap.ap_prefill(c, r, 0, GiB // page)
dcopy = torch.from_numpy(f).to("cuda")
out = torch.empty(grid * block, dtype=torch.int64, device="cuda")
out2 = torch.empty_like(out)
cfg = ap.bench_cfg(ap.AP_UNIFORM, 4, grid, block, reads_per_thread=reads, seed=11, span_bytes=GiB)
cfg_r = ap.bench_cfg(ap.AP_UNIFORM, 4, grid, block, reads_per_thread=reads, seed=11,
                     span_bytes=GiB, mode=ap.AP_MODE_RAW, raw_base=dcopy.data_ptr())


def t(fn, n=5):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(n):
        s.record()
        fn()
        e.record()
        e.synchronize()
        ts.append(s.elapsed_time(e) * 1e-3)
    return float(np.mean(ts))


st0 = ap.ap_cache_stats(c)
ta = t(lambda: ap.ap_bench_read(c, r, cfg, out))
st1 = ap.ap_cache_stats(c)
tr = t(lambda: ap.ap_bench_read(c, r, cfg_r, out2))
n = grid * block * reads
print(f"grid={grid} reads={n}: apointer {n / ta / 1e6:.1f} M reads/s, raw {n / tr / 1e6:.1f} M reads/s, "
      f"overhead {ta / tr - 1:+.3f}, equal={bool(torch.equal(out, out2))}, "
      f"majors={st1['major'] - st0['major']}, minors/launch={(st1['minor'] - st0['minor']) / 6:.0f}, "
      f"err={ap.ap_last_device_error(c)}")
