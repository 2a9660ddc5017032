"""A/B harness for the cache-hit regime (M2h) and the Fig. 6 per-access
workloads: apointer vs the raw twin at the same launch, median over
alternating launch pairs.  Env: AP_LIB_PATH (library variant),
AP_DEREF_GRIDS (comma list, default 296), AP_FIG6_TBS (default 148,296)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

GiB = 1 << 30
page, span, passes = 65536, GiB, 8
dev = torch.device("cuda:0")
raw = np.empty(2 * span + (1 << 21), np.uint8)
o = (-raw.ctypes.data) % (1 << 21)
f = synth.fill_file(raw[o:o + 2 * span], 1)
c = ap.ap_cache_create(2 * span // page + 16, page)
r = ap.ap_mmap(c, f)
ap.ap_prefill(c, r, 0, 2 * span // page)
dcopy = torch.from_numpy(f).to(dev)
torch.cuda.synchronize()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def t1(fn):
    s.record()
    fn()
    e.record()
    e.synchronize()
    return s.elapsed_time(e) * 1e-3


def pairs(fa, fr, n=8):
    for _ in range(2):
        fa()
        fr()
    ta, tr = [], []
    for _ in range(n):
        ta.append(t1(fa))
        tr.append(t1(fr))
    ta, tr = np.array(ta), np.array(tr)
    return float(np.median(ta)), float(np.median(tr)), float(np.median(ta / tr) - 1)


lib = os.path.basename(os.environ.get("AP_LIB_PATH", "default"))
nb = span * passes
for acc, name, grids in ((ap.AP_ACCESS_TILE, "tile", [148]), (ap.AP_ACCESS_RANGE, "range", [148]),
                         (ap.AP_ACCESS_DEREF, "deref",
                          [int(x) for x in os.environ.get("AP_DEREF_GRIDS", "296").split(",")])):
    for grid in grids:
        out = torch.empty(grid * 512, dtype=torch.int64, device=dev)
        out2 = torch.empty_like(out)
        cfg = ap.bench_cfg(ap.AP_SEQ, 16, grid, 512, unit_bytes=page, passes=passes, span_bytes=span,
                           access=acc)
        cfgr = ap.bench_cfg(ap.AP_SEQ, 16, grid, 512, unit_bytes=page, passes=passes,
                            span_bytes=span, mode=ap.AP_MODE_RAW, raw_base=dcopy.data_ptr(),
                            access=acc)
        ta, tr, ov = pairs(lambda: ap.ap_bench_read(c, r, cfg, out),
                           lambda: ap.ap_bench_read(c, r, cfgr, out2))
        print(f"{lib} {name:5s} grid {grid:4d}: apointer {nb / ta / 1e9:7.1f} GB/s  raw "
              f"{nb / tr / 1e9:7.1f} GB/s  overhead {100 * ov:+6.2f}%  equal "
              f"{bool(torch.equal(out, out2))}", flush=True)
for elem in (16, 4):
    for name in ("read", "add", "reduce", "fft", "bitonic"):
        for tb in [int(x) for x in os.environ.get("AP_FIG6_TBS", "148,296").split(",")]:
            out = torch.empty(tb * 512, dtype=torch.int64, device=dev)
            out2 = torch.empty_like(out)
            ta, tr, ov = pairs(lambda: ap.ap_bench_compute(c, r, name, elem, tb, 512, span, out),
                               lambda: ap.ap_bench_compute(c, r, name, elem, tb, 512, span, out2,
                                                           mode=ap.AP_MODE_RAW, raw_base=dcopy),
                               n=4)
            vb = (2 if name == "add" else 1) * span
            print(f"{lib} fig6 {elem:2d}B {name:7s} {tb:4d} TBs: apointer {vb / ta / 1e9:7.1f} GB/s "
                  f"raw {vb / tr / 1e9:7.1f} GB/s overhead {100 * ov:+6.1f}% equal "
                  f"{bool(torch.equal(out, out2))}", flush=True)
print(lib, "device error", ap.ap_last_device_error(c), ap.ap_cache_stats(c)["major"])
