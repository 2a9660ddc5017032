"""C5 partitions on one GPU: the collage's query blocks are
split into G contiguous ranges (mgpu.block_range), or -- with AP_SCHED_TABLE,
as bench.py --gpus G does -- the (table, bucket)-sorted units are
(mgpu.unit_range), and each rank's share is run ALONE on this GPU from a cold
2 GiB cache.  With
G GPUs each rank has its own page cache and its own host link, so the G-GPU
step time is max over ranks of these per-range times, provided the host's
memory system feeds G links at once (not measured here: one GPU per call).
Prints, per G: per-rank seconds, fills, and max / (T1 / G).

Usage: python tools/c5_partitions.py [schedule] [blocks|units|records] [id_chunks]
       (default: schedule 2 = AP_SCHED_TABLE, partitioned by units, 12 record-id
       windows per rank as bench.py's C5 default)"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench_collage as bc  # noqa: E402
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402
from paper_conf_isca_shaharbs16_b200 import mgpu  # noqa: E402

sched = int(sys.argv[1]) if len(sys.argv) > 1 else 2
cfg = bc.collage_config("c5")
dev = torch.device("cuda:0")
stream = torch.cuda.current_stream()
recs, keep = bc._shm_records(cfg, 0, 1, None)
img, _, _ = synth.make_target(cfg["W"], cfg["H"], cfg["N"], ds_seed=bc.DS_SEED, seed=bc.TGT_SEED,
                              pool=256, copy_permille=50)
proj, bias = synth.make_lsh_params(cfg["L"], cfg["K"], cfg["w"], seed=bc.LSH_SEED)
cache = ap.ap_cache_create(cfg["frames"], cfg["page"])
region = ap.ap_mmap(cache, recs)
B = 1 << cfg["bb"]
off = torch.empty((cfg["L"], B + 1), dtype=torch.int32, device=dev)
ids = torch.empty((cfg["L"], cfg["N"]), dtype=torch.int32, device=dev)
pd, bd = torch.from_numpy(proj).to(dev), torch.from_numpy(bias).to(dev)
ap.ap_lsh_build_index(cache, region, cfg["N"], cfg["stride"], cfg["L"], cfg["K"], cfg["bb"],
                      cfg["w"], pd, bd, off, ids)
tgt = torch.from_numpy(img).to(dev)
nb = (cfg["W"] // 32) * (cfg["H"] // 32)
full = None


def run_range(b0, b1, reps=2, u0=0, u1=0, i0=0, i1=0, nwin=None):
    inp = ap.collage_in(tgt, cfg["W"], cfg["H"], pd, bd, cfg["w"], cfg["bb"], off, ids, cfg["N"],
                        cfg["stride"], group=8, block_begin=b0, block_count=b1 - b0,
                        schedule=sched, unit_begin=u0, unit_count=u1 - u0,
                        id_chunks=(chunks if nwin is None else nwin) if sched in (2, 3) else 0,
                        id_begin=i0, id_end=i1)
    win = torch.empty((b1 - b0, 2), dtype=torch.int32, device=dev)
    ts = []
    for _ in range(reps):
        ap.ap_cache_reset(cache)
        torch.cuda.synchronize()
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(stream)
        ap.ap_collage_run(cache, region, inp, win, stream)
        e.record(stream)
        e.synchronize()
        ts.append(s.elapsed_time(e) * 1e-3)
    return min(ts), ap.ap_cache_stats(cache)["fill_bytes"], win


mode = sys.argv[2] if len(sys.argv) > 2 else ("units" if sched in (2, 3) else "blocks")
chunks = int(sys.argv[3]) if len(sys.argv) > 3 else 12
print(f"# C5 partitions run alone on one B200 (cold 2 GiB cache each), schedule {sched}, "
      f"partition by {mode}, {chunks} record-id windows; {nb} blocks, {cfg['N']} records")
flip = torch.tensor(-(1 << 63), dtype=torch.int64, device=dev)
t1 = None
for G in (1, 2, 4, 8):
    per, fills, parts = [], [], []
    for r in range(G):
        if mode == "units":  # rank r: a slice of the (table, bucket)-sorted units, all blocks
            u0, u1 = mgpu.unit_range(cfg["L"] * nb, r, G)
            t, fb, w = run_range(0, nb, u0=u0, u1=u1)
        elif mode == "records":  # rank r: all units, records [i0, i1) only
            i0, i1 = mgpu.id_range(cfg["N"], r, G)
            t, fb, w = run_range(0, nb, i0=i0, i1=i1, nwin=max(1, -(-chunks // G)))
        else:
            b0, b1 = mgpu.block_range(nb, r, G)
            t, fb, w = run_range(b0, b1)
        per.append(t)
        fills.append(fb)
        parts.append(w)
    if mode in ("units", "records"):  # the MIN reduction of reduce_winners_min, on one device
        acc = parts[0].view(torch.int64).view(-1) ^ flip
        for w in parts[1:]:
            acc = torch.minimum(acc, w.view(torch.int64).view(-1) ^ flip)
        whole = (acc ^ flip).view(torch.int32).view(-1, 2)
    else:
        whole = torch.cat(parts)
    if full is None:
        full = whole
    same = bool(torch.equal(whole, full))
    if t1 is None:
        t1 = per[0]
    tg = max(per)
    print(f"G={G}: per-rank s {[round(x, 4) for x in per]}  max {tg:.4f} s  "
          f"fills GB {[round(x / 1e9, 2) for x in fills]} (sum {sum(fills) / 1e9:.1f})  "
          f"T1/(G*max) = {t1 / (G * tg):.3f}  winners == G=1: {same}", flush=True)
print("device error", ap.ap_last_device_error(cache))
