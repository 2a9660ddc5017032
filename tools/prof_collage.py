"""Profiling harness: the collage on a fully resident page cache (every record
prefilled) -- apointer kernel vs its raw twin on an HBM copy, candidate
groupings 1/2/4 (the regime where apointer overhead is visible).
Prints CUDA-event timings; run under ncu for counters (-k regex:k_collage).

Usage: prof_collage.py [N_records] [group ...]      (default 1048576, 4)
Env:   AP_LIB_PATH selects a library variant; AP_PROF_STEPS timed repeats."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 20
groups = [int(g) for g in sys.argv[2:]] or [4]
steps = int(os.environ.get("AP_PROF_STEPS", 5))
W = H = 1024
stride_env = int(os.environ.get("AP_PROF_STRIDE", 4096))
L, K, bb, w, page, stride = 4, 8, 14, 60000, 4096, stride_env
dev = torch.device("cuda:0")
stream = torch.cuda.current_stream()

raw = np.empty(N * stride + (1 << 21), np.uint8)
o = (-raw.ctypes.data) % (1 << 21)
recs = synth.fill_records(raw[o:o + N * stride], 0, N, stride, 21)
img, _, _ = synth.make_target(W, H, N, ds_seed=21, seed=23, pool=256, copy_permille=50)
proj, bias = synth.make_lsh_params(L, K, w, seed=22)
npages = N * stride // page
cache = ap.ap_cache_create(npages + 64, page)
region = ap.ap_mmap(cache, recs)
off = torch.empty((L, (1 << bb) + 1), dtype=torch.int32, device=dev)
ids = torch.empty((L, N), dtype=torch.int32, device=dev)
pd, bd = torch.from_numpy(proj).to(dev), torch.from_numpy(bias).to(dev)
ap.ap_lsh_build_index(cache, region, N, stride, L, K, bb, w, pd, bd, off, ids)
tgt = torch.from_numpy(img).to(dev)
nb = (W // 32) * (H // 32)
# cold run on a cache that holds every record: majors = distinct records touched
ic = ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, N, stride, group=groups[0], block_begin=0,
                   block_count=nb)
wc = torch.empty((nb, 2), dtype=torch.int32, device=dev)
ap.ap_cache_reset(cache)
ap.ap_collage_run(cache, region, ic, wc, stream)
torch.cuda.synchronize()
print(f"distinct records touched (cold, cache >= file): {ap.ap_cache_stats(cache)['major']}", flush=True)
ap.ap_cache_reset(cache)
ap.ap_prefill(cache, region, 0, npages, stream)
dcopy = torch.from_numpy(recs).to(dev)
torch.cuda.synchronize()


def timed(fn):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(steps):
        s.record(stream)
        fn()
        e.record(stream)
        e.synchronize()
        ts.append(s.elapsed_time(e) * 1e-3)
    return min(ts)


for sched in [int(x) for x in os.environ.get("AP_PROF_SCHEDS", "1,0").split(",")]:
    for g in groups:
        mk = lambda mode, rb: ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, N, stride, group=g,  # noqa: E731
                                            block_begin=0, block_count=nb, mode=mode, raw_base=rb,
                                            schedule=sched)
        ia, ir = mk(ap.AP_MODE_APOINTER, None), mk(ap.AP_MODE_RAW, dcopy)
        wa = torch.empty((nb, 2), dtype=torch.int32, device=dev)
        wr = torch.empty_like(wa)
        ap.ap_collage_run(cache, region, ia, wa, stream)
        ap.ap_collage_run(cache, region, ir, wr, stream)
        torch.cuda.synchronize()
        ta = timed(lambda: ap.ap_collage_run(cache, region, ia, wa, stream))
        tr = timed(lambda: ap.ap_collage_run(cache, region, ir, wr, stream))
        st = ap.ap_cache_stats(cache)
        print(f"N={N} sched={sched} group={g} apointer {ta*1e3:.3f} ms raw {tr*1e3:.3f} ms "
              f"overhead {ta/tr-1:+.3f} equal={bool(torch.equal(wa, wr))} majors={st['major']} "
              f"minors={st['minor']} err={ap.ap_last_device_error(cache)}", flush=True)
ap.ap_munmap(cache, region)
ap.ap_cache_destroy(cache)
