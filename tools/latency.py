"""Table I analogue on B200: cycles per 4-B read / pointer
increment, raw vs apointer, one warp, coalesced, one page."""
import sys

import numpy as np

sys.path.insert(0, ".")
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

raw = np.empty((1 << 20) + 4096, np.uint8)
o = (-raw.ctypes.data) % 4096
f = synth.fill_file(raw[o:o + (1 << 20)], 1)
names = ["read", "apointer read", "inc", "apointer inc", "read+inc", "apointer read+inc"]
print("# B200 latency (clock64 cycles per op, 1 warp, coalesced 4-B, one page; empty timing pair subtracted)")
for page in (4096, 65536):
    c = ap.ap_cache_create(8, page)
    r = ap.ap_mmap(c, f)
    res = {}
    for op in range(6):
        cyc, empty = ap.ap_bench_latency(c, r, op, 2000)
        res[names[op]] = cyc
    print(f"page={page}: " + ", ".join(f"{k}={v}" for k, v in res.items()) + f" (empty pair={empty})")
    for a, b in (("read", "apointer read"), ("inc", "apointer inc"), ("read+inc", "apointer read+inc")):
        base = max(res[a], 1)
        print(f"   {b}: {res[b]} vs {res[a]} ({(res[b] - res[a]) / base * 100:+.0f}%)")
    ap.ap_munmap(c, r)
    ap.ap_cache_destroy(c)
