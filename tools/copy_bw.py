"""Table II analogue: copy between two regions through
apointers (tiled reads, per-element stores), pages resident, vs the same bytes
copied device-to-device by cudaMemcpy (torch copy_)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

GiB = 1 << 30
span = GiB // 2
page = 65536
raw = np.empty(2 * span + (1 << 21), np.uint8)
o = (-raw.ctypes.data) % (1 << 21)
src = synth.fill_file(raw[o:o + span], 1)
dst = raw[o + span:o + 2 * span]
dst[:] = 0
c = ap.ap_cache_create(2 * span // page + 64, page)
rs = ap.ap_mmap(c, src)
rd = ap.ap_mmap_prot(c, dst, ap.AP_PROT_READ | ap.AP_PROT_WRITE)
ap.ap_prefill(c, rs, 0, span // page)
ap.ap_prefill(c, rd, 0, span // page)
torch.cuda.synchronize()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def t(fn, n=5):
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


a = torch.empty(span, dtype=torch.uint8, device="cuda")
b = torch.empty_like(a)
tm = t(lambda: b.copy_(a))
print(f"# B200 copy bandwidth (read+write bytes / time), {span >> 20} MiB, pages resident")
print(f"cudaMemcpy D2D (torch copy_): {2 * span / tm / 1e9:.1f} GB/s")
both = torch.empty(2 * span, dtype=torch.uint8, device="cuda")
both[:span].copy_(torch.from_numpy(src))
import os  # noqa: E402
grid = int(os.environ.get("AP_GRID", 148))
for elem in (4, 8, 16):
    cfg = ap.bench_cfg(ap.AP_SEQ, elem, grid, 512, unit_bytes=page, span_bytes=span)
    cfg_r = ap.bench_cfg(ap.AP_SEQ, elem, grid, 512, unit_bytes=page, span_bytes=span,
                         mode=ap.AP_MODE_RAW, raw_base=both.data_ptr())
    ta = t(lambda: ap.ap_bench_copy(c, rs, rd, cfg))
    tr = t(lambda: ap.ap_bench_copy(c, rs, rd, cfg_r))
    print(f"apointer copy {elem:2d}-B: {2 * span / ta / 1e9:.1f} GB/s "
          f"({tm / ta * 100:.1f}% of cudaMemcpy); raw twin (same loop) {2 * span / tr / 1e9:.1f} GB/s "
          f"({tm / tr * 100:.1f}%), apointer overhead {ta / tr - 1:+.3f}")
assert torch.equal(both[span:], both[:span]), "raw twin copy wrong"
print("device error", ap.ap_last_device_error(c))
ap.ap_munmap(c, rd)
ap.ap_munmap(c, rs)
print("dst == src after write-back:", bool(np.array_equal(dst, src)))
