"""Hash-table page table (N4 ablation) repro: the DIVERGENT cold case of
test_link_events_closed_form, values vs the oracle, device error word."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import oracle  # noqa: E402
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
from helpers import check_invariants, make_file  # noqa: E402

print(ap.ap_version())
for nbytes, page, frames_extra, grid in [(16 << 20, 4096, 8, 4), (64 << 20, 4096, 8, 8),
                                         (256 << 20, 4096, 8, 32), (256 << 20, 4096, -60000, 32)]:
    f = make_file(nbytes, seed=31)
    npages = nbytes // page
    frames = npages + frames_extra
    c = ap.ap_cache_create(frames, page)
    r = ap.ap_mmap(c, f)
    block, reads, seed = 256, 4, 77
    n = grid * block
    out = torch.zeros(n, dtype=torch.int64, device="cuda")
    cfg = ap.bench_cfg(2, 4, grid, block, reads_per_thread=reads, seed=seed, page_bytes=page)
    ap.ap_bench_read(c, r, cfg, out)
    torch.cuda.synchronize()
    err = ap.ap_last_device_error(c)
    got = out.cpu().numpy().view(np.uint64)
    want = oracle.read_divergent(f, nbytes, page, 4, n, reads, seed)
    bad = np.nonzero(got != want)[0]
    print(f"nbytes={nbytes >> 20} MiB frames={frames} grid={grid}: err={err} wrong threads={len(bad)}"
          f" first={bad[:8].tolist()} stats={ap.ap_cache_stats(c)}", flush=True)
    print("  invariants:", check_invariants(ap, c, [r], frames)[:4], flush=True)
    ap.ap_munmap(c, r)
    ap.ap_cache_destroy(c)
