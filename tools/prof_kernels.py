"""Profiling harness for the hit-regime kernels: one launch each, in this
order, over a resident GiB (64 KiB pages, 16-B reads unless noted):
  k_seq        apointer tile, raw tile           (M2h, the tiled form)
  k_seq_deref  apointer per-access, raw twin     (M2h, `v = *q; q += 32`)
  k_random     apointer M2r, raw gather          (uniform 4-B, every read a link)
Run under ncu with -k regex:'^k_seq$' (etc.) -c 2.  Env: AP_LIB_PATH."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

GiB = 1 << 30
page, span = 65536, GiB
dev = torch.device("cuda:0")
raw = np.empty(span + (1 << 21), np.uint8)
o = (-raw.ctypes.data) % (1 << 21)
f = synth.fill_file(raw[o:o + span], 1)
c = ap.ap_cache_create(span // page + 16, page)
r = ap.ap_mmap(c, f)
ap.ap_prefill(c, r, 0, span // page)
dcopy = torch.from_numpy(f).to(dev)
torch.cuda.synchronize()
runs = [("tile", ap.AP_SEQ, 16, 148, dict(unit_bytes=page, passes=2, access=ap.AP_ACCESS_TILE)),
        ("deref", ap.AP_SEQ, 16, 148, dict(unit_bytes=page, passes=2, access=ap.AP_ACCESS_DEREF)),
        ("minor", ap.AP_UNIFORM, 4, 592, dict(reads_per_thread=8, seed=11))]
for name, pat, elem, grid, kw in runs:
    outs = []
    for mode in (ap.AP_MODE_APOINTER, ap.AP_MODE_RAW):
        extra = dict(mode=mode, raw_base=dcopy.data_ptr()) if mode == ap.AP_MODE_RAW else {}
        cfg = ap.bench_cfg(pat, elem, grid, 512, span_bytes=span, **kw, **extra)
        out = torch.empty(grid * 512, dtype=torch.int64, device=dev)
        ap.ap_bench_read(c, r, cfg, out)
        outs.append(out)
    torch.cuda.synchronize()
    print(name, "equal", bool(torch.equal(outs[0], outs[1])), flush=True)
print("err", ap.ap_last_device_error(c))
