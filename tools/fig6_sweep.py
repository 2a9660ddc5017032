"""Fig. 6a/6b analogue: apointer overhead over the raw
twin for the compute-intensity workloads as a function of occupancy (thread
blocks of 512 threads), 4-B and 16-B loads, pages resident (no faults)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

page = 65536
span = 1 << 30
raw = np.empty(2 * span + (1 << 21), np.uint8)
o = (-raw.ctypes.data) % (1 << 21)
f = synth.fill_file(raw[o:o + 2 * span], 1)
c = ap.ap_cache_create(2 * span // page + 16, page)
r = ap.ap_mmap(c, f)
ap.ap_prefill(c, r, 0, 2 * span // page)
dcopy = torch.from_numpy(f).to("cuda")
torch.cuda.synchronize()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def timed(fn, n=3):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(n):
        s.record()
        fn()
        e.record()
        e.synchronize()
        ts.append(s.elapsed_time(e))
    return float(np.mean(ts))


works = [("add", 0), ("read", 0), ("random", 10), ("random", 50), ("reduce", 0), ("fft", 0),
         ("bitonic", 0)]
import os
MINB = int(os.environ.get("AP_FIG6_MINB", 1))  # CTAs of 512 per SM the library's k_compute is built for
tbs = [t for t in (1, 4, 16, 37, 74, 148, 296, 444, 592) if t <= 148 * MINB]
print("# apointer overhead vs raw twin (time_ap / time_raw - 1), 512-thread blocks, "
      f"{span >> 20} MiB per vector resident, one access at a time (no tiling)")
for elem in (4, 16):
    print(f"\n## {elem}-byte loads (Fig. 6{'a' if elem == 4 else 'b'} analogue)")
    print("workload      " + "".join(f"{t:>8d}TB" for t in tbs))
    for name, it in works:
        row = []
        for tb in tbs:
            out = torch.empty(tb * 512, dtype=torch.int64, device="cuda")
            out2 = torch.empty_like(out)
            ta = timed(lambda: ap.ap_bench_compute(c, r, name, elem, tb, 512, span, out, iters=it))
            tr = timed(lambda: ap.ap_bench_compute(c, r, name, elem, tb, 512, span, out2, iters=it,
                                                   mode=ap.AP_MODE_RAW, raw_base=dcopy))
            assert torch.equal(out, out2)
            row.append(ta / tr - 1)
        label = f"{name}-{it}" if name == "random" else name
        print(f"{label:13s} " + "".join(f"{100 * v:9.1f}%" for v in row))
print("\ndevice error", ap.ap_last_device_error(c))
