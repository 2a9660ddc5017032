"""C1 (16 MiB, 4 KiB pages, 64 frames, 148 warps) under different back-off caps."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402
n = 16 << 20
raw = np.empty(n + 4096, np.uint8); o = (-raw.ctypes.data) % 4096
f = synth.fill_file(raw[o:o + n], 1)
c = ap.ap_cache_create(64, 4096)
r = ap.ap_mmap(c, f)
out = torch.empty(n, dtype=torch.uint8, device="cuda")
cfg = ap.bench_cfg(ap.AP_SEQ, 16, 148, 32, unit_bytes=4096, out_copy=True)
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for mn, mx in ((64, 4096), (64, 1024), (32, 256), (16, 64)):
    for steps in (64, 4):
        ap.ap_cache_set_backoff(c, mn, mx)
        ap.ap_cache_set_tuning(c, 1, steps, 0)
        ts = []
        for i in range(6):
            ap.ap_cache_reset(c)
            s.record(); ap.ap_bench_read(c, r, cfg, out); e.record(); e.synchronize()
            if i >= 2: ts.append(s.elapsed_time(e))
        st = ap.ap_cache_stats(c)
        ok = bool(np.array_equal(out.cpu().numpy(), f))
        print(f"backoff {mn}-{mx} ns sweep_steps {steps}: {np.mean(ts):.3f} ms  fill {st['fill_bytes'] / (np.mean(ts) * 1e-3) / 1e9:.2f} GB/s  waits {st['waits']} nofree {st['nofree']} ok={ok}")
