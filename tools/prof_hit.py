"""Profiling harness: cache-hit mode (M2h) apointer kernel and its raw twin,
plus (optionally) the C2 fault-bound kernel.  Prints event timings; run under
ncu for counters.  Usage: prof_hit.py [unit_bytes] [passes] [c2]"""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

GiB = 1 << 30
unit = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
passes = int(sys.argv[2]) if len(sys.argv) > 2 else 8
do_c2 = len(sys.argv) > 3 and sys.argv[3] == "c2"
dev = torch.device("cuda:0")
span = GiB
fbytes = 4 * GiB if do_c2 else span
raw = np.empty(fbytes + (1 << 21), np.uint8)
o = (-raw.ctypes.data) % (1 << 21)
f = synth.fill_file(raw[o:o + fbytes], 1)
cache = ap.ap_cache_create(16384, 65536)
r = ap.ap_mmap(cache, f)
ap.ap_prefill(cache, r, 0, span // 65536)
torch.cuda.synchronize()
import os
grid, block = int(os.environ.get("AP_GRID", 148)), int(os.environ.get("AP_BLOCK", 512))
out = torch.empty(grid * block, dtype=torch.int64, device=dev)
out2 = torch.empty_like(out)
dcopy = torch.from_numpy(f[:span]).to(dev)
cfg = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=unit, passes=passes, span_bytes=span)
cfg_raw = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=unit, passes=passes,
                       span_bytes=span, mode=ap.AP_MODE_RAW, raw_base=dcopy.data_ptr())


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
    return min(ts), float(np.mean(ts))


tr = t(lambda: ap.ap_bench_read(cache, r, cfg_raw, out2))
nb = span * passes
cfg_traw = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=unit, passes=passes, span_bytes=span,
                        mode=ap.AP_MODE_RAW, raw_base=dcopy.data_ptr(), access=ap.AP_ACCESS_TMA)
cfg_tap = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=unit, passes=passes, span_bytes=span,
                       access=ap.AP_ACCESS_TMA)
out3 = torch.empty_like(out)
for _ in range(3):
    ttr = t(lambda: ap.ap_bench_read(cache, r, cfg_traw, out3))
    tta = t(lambda: ap.ap_bench_read(cache, r, cfg_tap, out))
    print(f"unit={unit} passes={passes} tma   apointer {span * passes / tta[1] / 1e9:.1f} GB/s raw-tma "
          f"{span * passes / ttr[1] / 1e9:.1f} GB/s overhead {tta[1] / ttr[1] - 1:.3f} "
          f"(vs tiled raw {tta[1] / tr[1] - 1:+.3f}) equal={bool(torch.equal(out, out2)) and bool(torch.equal(out3, out2))}")
for acc, name in ((ap.AP_ACCESS_TILE, "tile"), (ap.AP_ACCESS_AHEAD, "ahead"), (ap.AP_ACCESS_PAIR, "pair"), (ap.AP_ACCESS_RANGE, "range"), (ap.AP_ACCESS_DEREF, "deref")):
    cfg = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=unit, passes=passes, span_bytes=span,
                       access=acc)
    ta = t(lambda: ap.ap_bench_read(cache, r, cfg, out))
    print(f"unit={unit} passes={passes} {name:5s} apointer {nb/ta[1]/1e9:.1f} GB/s raw {nb/tr[1]/1e9:.1f} GB/s "
          f"overhead {ta[1]/tr[1]-1:.3f} equal={bool(torch.equal(out, out2))}")
if do_c2:
    cfg2 = ap.bench_cfg(ap.AP_UNIFORM, 4, 148, 512, reads_per_thread=8, seed=1234)
    ap.ap_cache_reset(cache)
    s = time.time()
    ap.ap_bench_read(cache, r, cfg2, out)
    torch.cuda.synchronize()
    st = ap.ap_cache_stats(cache)
    print("c2", time.time() - s, st)
