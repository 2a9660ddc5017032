"""Profiling harness for the per-access dereference (M2h, AP_ACCESS_DEREF)
and the Fig. 6 Read workload: one warm-up and one profiled launch each of the
apointer kernel and its raw twin over a resident GiB.  Run under ncu with
-k regex:'k_seq_deref|k_compute'.  Env: AP_LIB_PATH, AP_GRID (default 592)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

GiB = 1 << 30
page, span = 65536, GiB
grid = int(os.environ.get("AP_GRID", 592))
dev = torch.device("cuda:0")
raw = np.empty(span + (1 << 21), np.uint8)
o = (-raw.ctypes.data) % (1 << 21)
f = synth.fill_file(raw[o:o + span], 1)
c = ap.ap_cache_create(span // page + 16, page)
r = ap.ap_mmap(c, f)
ap.ap_prefill(c, r, 0, span // page)
dcopy = torch.from_numpy(f).to(dev)
out = torch.empty(grid * 512, dtype=torch.int64, device=dev)
out2 = torch.empty_like(out)
cfg = ap.bench_cfg(ap.AP_SEQ, 16, grid, 512, unit_bytes=page, passes=2, span_bytes=span,
                   access=ap.AP_ACCESS_DEREF)
cfgr = ap.bench_cfg(ap.AP_SEQ, 16, grid, 512, unit_bytes=page, passes=2, span_bytes=span,
                    access=ap.AP_ACCESS_DEREF, mode=ap.AP_MODE_RAW, raw_base=dcopy.data_ptr())
for _ in range(2):
    ap.ap_bench_read(c, r, cfg, out)
    ap.ap_bench_read(c, r, cfgr, out2)
torch.cuda.synchronize()
print("equal", bool(torch.equal(out, out2)), "err", ap.ap_last_device_error(c))
