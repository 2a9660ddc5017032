"""Collage workloads for bench.py (--workload c4 | c5): PAPER.md:405-442.

C4 (BASELINE configs[3]): 1M 32x32 tiles (4 GiB file of 4 KiB-padded
histograms), 1024x1024 target, LSH candidate lists, integer SSD, 1 B200.
C5 (configs[4]): 10M tiles (40.96 GB pinned host file), 8192x8192 target,
query blocks partitioned over the ranks, each with its own 2 GiB page cache,
one NCCL gather of the per-block winners to rank 0.

A step = reset the cache (cold, untimed), then the collage kernel over this
rank's block range (+ the gather when N > 1), timed with CUDA events on the
launch stream; the step time is the max over ranks.
"""
import json
import mmap
import os
import time

import numpy as np

GiB = 1 << 30
SCHED_NAMES = {0: "natural order (one CTA per block, the paper's single kernel)",
               1: "lsh-sorted blocks", 2: "per-table units sorted by (table, bucket)",
               3: "per-table units sorted by (bucket MinHash, table, bucket)"}
LSH_SEED, DS_SEED, TGT_SEED = 22, 21, 23


def collage_config(name, stride=4096):
    cfg = _collage_config(name)
    if os.environ.get("AP_COLLAGE_FRAMES"):  # experiments only (e.g. a cache >= the file)
        cfg["frames"] = int(os.environ["AP_COLLAGE_FRAMES"])
        cfg["workload"] += f"; CACHE OVERRIDE {cfg['frames']} frames"
    if stride != 4096:  # NEXT N1: unaligned 3 KiB records, no padding
        cfg["stride"] = stride
        cfg["workload"] += f"; UNALIGNED {stride}-B records (no padding, records straddle pages)"
    return cfg


def _collage_config(name):
    if name == "c4":
        return dict(name="c4", N=1 << 20, W=1024, H=1024, L=4, K=8, bb=14, w=60000,
                    frames=65536, page=4096, stride=4096,
                    workload="C4: 1M 32x32 RGB tiles (4 GiB file of 4 KiB-padded histograms in "
                             "pinned host memory), 1024x1024 target, LSH L=4 K=8 2^14 buckets, "
                             "integer SSD, 256 MiB page cache (cold per step), 1 B200")
    return dict(name="c5", N=10_000_000, W=8192, H=8192, L=4, K=8, bb=16, w=40000,
                frames=524288, page=4096, stride=4096,
                workload="C5: 10M tiles in a 40.96 GB pinned host file, 8192x8192 target, LSH "
                         "L=4 K=8 2^16 buckets, work partitioned over the ranks (--partition), 2 "
                         "GiB page cache per GPU (cold per step); N > 1: winners folded into rank "
                         "0's array by the kernels (--combine fused) or one NCCL gather / MIN "
                         "reduce (--combine nccl)")


def numa_interleave(arr):
    """Spread the pages of a host buffer round-robin over the host's NUMA
    nodes (mbind MPOL_INTERLEAVE before the first touch), so G GPUs reading
    the one pinned file over their own PCIe links do not all pull from the
    memory of one socket (SURVEY.md §7 "Host side at scale").  Returns the
    node count used (1 = nothing to do or not supported)."""
    import ctypes
    try:
        with open("/sys/devices/system/node/online") as f:
            spec = f.read().strip()
        nodes = []
        for part in spec.split(","):
            a, _, b = part.partition("-")
            nodes.extend(range(int(a), int(b or a) + 1))
    except OSError:
        return 1
    if len(nodes) < 2:
        return 1
    mask = 0
    for n in nodes:
        mask |= 1 << n
    libc = ctypes.CDLL(None, use_errno=True)
    page = 4096
    addr = arr.ctypes.data & ~(page - 1)
    length = arr.ctypes.data + arr.nbytes - addr
    nm = ctypes.c_ulong(mask)
    SYS_mbind, MPOL_INTERLEAVE = 237, 3  # x86_64
    rc = libc.syscall(SYS_mbind, ctypes.c_void_p(addr), ctypes.c_ulong(length), MPOL_INTERLEAVE,
                      ctypes.byref(nm), ctypes.c_ulong(max(nodes) + 2), 0)
    return len(nodes) if rc == 0 else 1


def _shm_records(cfg, rank, world, dist):
    """The record file in /dev/shm, generated once (all ranks map the same
    pages; each rank registers them for its own GPU)."""
    import synth
    nbytes = cfg["N"] * cfg["stride"]
    path = f"/dev/shm/apb_{cfg['name']}_{cfg['N']}_{cfg['stride']}_{DS_SEED}.bin"
    done = path + ".ok"
    if rank == 0 and os.environ.get("AP_REUSE_SHM") != "1":
        # a file left by an earlier process is not reused (a timing must not
        # depend on what ran before on the box); AP_REUSE_SHM=1 keeps it
        for f_ in (done, path):
            if os.path.exists(f_):
                os.remove(f_)
    if rank == 0 and not os.path.exists(done):
        with open(path, "wb") as fh:
            fh.truncate(nbytes)
        with open(path, "r+b") as fh:
            mm = mmap.mmap(fh.fileno(), nbytes)
            arr = np.frombuffer(mm, dtype=np.uint8)
            numa_interleave(arr)  # before the first touch
            chunk = 1 << 18
            for first in range(0, cfg["N"], chunk):
                cnt = min(chunk, cfg["N"] - first)
                synth.fill_records(arr[first * cfg["stride"]:(first + cnt) * cfg["stride"]], first,
                                   cnt, cfg["stride"], DS_SEED)
            del arr
            mm.flush()
            mm.close()
        open(done, "w").close()
    if dist is not None:
        dist.barrier()
    fh = open(path, "r+b")
    mm = mmap.mmap(fh.fileno(), nbytes)
    return np.frombuffer(mm, dtype=np.uint8), (fh, mm)


def run_collage(args, torch, dev, rank, world, dist, timed, ClockSampler, host_link_peak,
                light=False):
    import paper_conf_isca_shaharbs16_b200 as ap
    import synth
    cfg = collage_config(args.workload, args.stride)
    stream = torch.cuda.current_stream()
    t0 = time.time()
    if cfg["name"] == "c4":
        from bench import aligned_empty
        recs = synth.fill_records(aligned_empty(cfg["N"] * cfg["stride"]), 0, cfg["N"],
                                  cfg["stride"], DS_SEED)
        keep = None
    else:
        recs, keep = _shm_records(cfg, rank, world, dist)
    img, src, is_copy = synth.make_target(cfg["W"], cfg["H"], cfg["N"], ds_seed=DS_SEED,
                                          seed=TGT_SEED, pool=256, copy_permille=50)
    proj, bias = synth.make_lsh_params(cfg["L"], cfg["K"], cfg["w"], seed=LSH_SEED)
    t_gen = time.time() - t0
    cache = ap.ap_cache_create(cfg["frames"], cfg["page"], torch.cuda.current_device())
    t0 = time.time()
    region = ap.ap_mmap(cache, recs)
    t_pin = time.time() - t0
    B = 1 << cfg["bb"]
    off = torch.empty((cfg["L"], B + 1), dtype=torch.int32, device=dev)
    ids = torch.empty((cfg["L"], cfg["N"]), dtype=torch.int32, device=dev)
    pd, bd = torch.from_numpy(proj).to(dev), torch.from_numpy(bias).to(dev)
    t0 = time.time()
    ap.ap_lsh_build_index(cache, region, cfg["N"], cfg["stride"], cfg["L"], cfg["K"], cfg["bb"],
                          cfg["w"], pd, bd, off, ids)
    t_index = time.time() - t0
    nb = (cfg["W"] // 32) * (cfg["H"] // 32)
    from paper_conf_isca_shaharbs16_b200 import mgpu
    # N > 1: AP_SCHED_TABLE splits the (table, bucket)-sorted units (each
    # bucket read by one rank, winners MIN-reduced); the other schedules split
    # the image into block ranges (winners gathered)
    # --partition records: every rank runs all units over its slice of the
    # record ids (each GPU caches one shard of the file), winners MIN-reduced
    part = args.partition if args.schedule in (2, 3) else "blocks"
    bucket = part in ("units", "records") and world > 1
    i0, i1 = 0, 0
    if bucket and part == "records":
        b0, b1 = 0, nb
        u0, u1 = 0, 0
        i0, i1 = mgpu.id_range(cfg["N"], rank, world)
    elif bucket:
        b0, b1 = 0, nb
        u0, u1 = mgpu.unit_range(cfg["L"] * nb, rank, world)
    else:
        b0, b1 = mgpu.block_range(nb, rank, world)
        u0, u1 = 0, 0
    tgt_host = torch.from_numpy(img).pin_memory()
    tgt = tgt_host.to(dev)
    win = torch.empty((b1 - b0, 2), dtype=torch.int32, device=dev)
    id_chunks = args.id_chunks if args.id_chunks is not None else {"c4": 32, "c5": 96}.get(cfg["name"], 0)
    id_chunks = id_chunks if args.schedule in (2, 3) else 0
    if i1:  # the windows split this rank's record slice
        id_chunks = max(1, -(-id_chunks // world))
    inp = ap.collage_in(tgt, cfg["W"], cfg["H"], pd, bd, cfg["w"], cfg["bb"], off, ids, cfg["N"],
                        cfg["stride"], group=args.group, block_begin=b0, block_count=b1 - b0,
                        schedule=args.schedule, unit_begin=u0, unit_count=u1 - u0,
                        id_chunks=id_chunks, id_begin=i0, id_end=i1)

    # N > 1, fused (default): every rank's kernel folds its winners into rank
    # 0's array over NVLink (CUDA IPC + system-scope atomic min), no
    # collective; --combine nccl: one NCCL gather / MIN reduce after the kernel
    fused = world > 1 and getattr(args, "combine", "fused") == "fused"
    sw = mgpu.SharedWinners(ap, nb, rank, world, dist, dev) if fused else None
    inp_f = None
    if fused:
        inp_f = ap.collage_in(tgt, cfg["W"], cfg["H"], pd, bd, cfg["w"], cfg["bb"], off, ids,
                              cfg["N"], cfg["stride"], group=args.group, block_begin=b0,
                              block_count=b1 - b0, schedule=args.schedule, unit_begin=u0,
                              unit_count=u1 - u0, id_chunks=id_chunks, id_begin=i0, id_end=i1,
                              flags=ap.AP_COLLAGE_ACCUMULATE | ap.AP_COLLAGE_SYSTEM)

    def combine():
        if fused:
            return sw.result
        if bucket:
            return mgpu.reduce_winners_min(win, rank, world, dist)  # one NCCL reduce (S12)
        return mgpu.gather_winners(win, rank, world, dist, nb)  # one NCCL gather (S12)

    def step():
        if fused:
            ap.ap_collage_run(cache, region, inp_f, sw.ptr(b0), stream)
            return
        ap.ap_collage_run(cache, region, inp, win, stream)
        if world > 1:
            combine()

    link = host_link_peak(torch, dev)
    for _ in range(args.warmup):
        ap.ap_cache_reset(cache)
        if fused:
            sw.begin(stream)
        elif world > 1:
            dist.barrier()
        timed(torch, step, stream)
        if fused:
            sw.end()
    times, stats = [], []
    with ClockSampler(torch.cuda.current_device()) as clk:
        for _ in range(args.steps):
            ap.ap_cache_reset(cache)  # cold cache each step (untimed)
            if fused:
                sw.begin(stream)  # rank 0 sets the sentinels; all ranks start together
            elif world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            times.append(timed(torch, step, stream))
            if fused:
                sw.end()  # every rank's folds are in rank 0's array
            stats.append(ap.ap_cache_stats(cache))
    if fused:
        # this rank's own share, for the comparisons below
        ap.ap_cache_reset(cache)
        ap.ap_collage_run(cache, region, inp, win, stream)
        torch.cuda.synchronize()
    err = ap.ap_last_device_error(cache)
    got = win.cpu().numpy().view(np.uint32).copy()
    # the other schedules, for comparison (cold cache, same winners)
    other_res = []
    for other in (s for s in (0, 1, 2, 3) if s != args.schedule and world == 1 and not light):
        inp_o = ap.collage_in(tgt, cfg["W"], cfg["H"], pd, bd, cfg["w"], cfg["bb"], off, ids,
                              cfg["N"], cfg["stride"], group=args.group, block_begin=b0,
                              block_count=b1 - b0, schedule=other)
        win_o = torch.empty_like(win)
        t_other = []
        for _ in range(2):
            ap.ap_cache_reset(cache)
            t_other.append(timed(torch, lambda: ap.ap_collage_run(cache, region, inp_o, win_o,
                                                                  stream), stream))
        other_stats = ap.ap_cache_stats(cache)
        other_res.append(dict(schedule=SCHED_NAMES[other], s=min(t_other),
                              major=other_stats["major"], fill_GB=other_stats["fill_bytes"] / 1e9,
                              equal=bool(torch.equal(win_o, win))))

    # raw twin: identical kernel on a fully resident HBM copy (c4 only: 4 GiB)
    raw = None
    if cfg["name"] == "c4":
        dcopy = torch.from_numpy(recs).to(dev)
        inp_raw = ap.collage_in(tgt, cfg["W"], cfg["H"], pd, bd, cfg["w"], cfg["bb"], off, ids,
                                        cfg["N"], cfg["stride"], group=args.group, block_begin=b0,
                                block_count=b1 - b0, mode=ap.AP_MODE_RAW, raw_base=dcopy,
                                schedule=args.schedule, unit_begin=u0, unit_count=u1 - u0,
                                id_begin=i0, id_end=i1)  # this rank's share, like inp
        win_raw = torch.empty_like(win)
        for _ in range(2):
            timed(torch, lambda: ap.ap_collage_run(cache, region, inp_raw, win_raw, stream), stream)
        raw_t = min(timed(torch, lambda: ap.ap_collage_run(cache, region, inp_raw, win_raw, stream),
                          stream) for _ in range(args.steps))
        # apointer on the warm (fully resident would need 4 GiB of frames) cache:
        # run the apointer kernel again without reset = warm-cache time
        warm_t = min(timed(torch, lambda: ap.ap_collage_run(cache, region, inp, win, stream),
                           stream) for _ in range(args.steps))
        raw = dict(raw_s=raw_t, warm_s=warm_t, equal=bool(torch.equal(win_raw, win)))
        # resident regime (the paper's "apointers vs GPUfs" comparison,
        # PAPER.md:440): a second cache that holds every record, prefilled;
        # apointer collage vs the raw twin, per candidate grouping
        npages = (cfg["N"] * cfg["stride"] + cfg["page"] - 1) // cfg["page"]
        big = ap.ap_cache_create(npages + 64, cfg["page"], torch.cuda.current_device())
        rb = ap.ap_mmap(big, recs)
        # one cold run on a cache that holds every record: its major faults
        # are the distinct record pages this rank's share touches, the
        # host-link lower bound of a cold step (each needed page read once)
        wd = torch.empty_like(win)
        ap.ap_collage_run(big, rb, inp, wd, stream)
        torch.cuda.synchronize()
        raw_distinct = ap.ap_cache_stats(big)["major"]
        ap.ap_cache_reset(big)
        ap.ap_prefill(big, rb, 0, npages, stream)
        torch.cuda.synchronize()
        res_g = {}
        for g in (1, 2, 4, 8):
            inp_g = ap.collage_in(tgt, cfg["W"], cfg["H"], pd, bd, cfg["w"], cfg["bb"], off, ids,
                                  cfg["N"], cfg["stride"], group=g, block_begin=b0,
                                  block_count=b1 - b0, schedule=args.schedule, unit_begin=u0,
                                  unit_count=u1 - u0, id_begin=i0, id_end=i1)
            inp_gr = ap.collage_in(tgt, cfg["W"], cfg["H"], pd, bd, cfg["w"], cfg["bb"], off, ids,
                                   cfg["N"], cfg["stride"], group=g, block_begin=b0,
                                   block_count=b1 - b0, mode=ap.AP_MODE_RAW, raw_base=dcopy,
                                   schedule=args.schedule, unit_begin=u0, unit_count=u1 - u0,
                                   id_begin=i0, id_end=i1)
            wg, wr = torch.empty_like(win), torch.empty_like(win)
            for _ in range(2):
                ap.ap_collage_run(big, rb, inp_g, wg, stream)
                ap.ap_collage_run(big, rb, inp_gr, wr, stream)
            ta = min(timed(torch, lambda: ap.ap_collage_run(big, rb, inp_g, wg, stream), stream)
                     for _ in range(args.steps))
            tr = min(timed(torch, lambda: ap.ap_collage_run(big, rb, inp_gr, wr, stream), stream)
                     for _ in range(args.steps))
            res_g[g] = dict(apointer_s=ta, raw_s=tr, overhead=ta / tr - 1,
                            equal=bool(torch.equal(wg, win) and torch.equal(wr, win)))
        raw["resident"] = res_g
        raw["resident_majors"] = ap.ap_cache_stats(big)["major"]
        raw["distinct_pages"] = raw_distinct
        raw["distinct_equal"] = bool(torch.equal(wd, win))
        ap.ap_munmap(big, rb)
        ap.ap_cache_destroy(big)
        del dcopy

    # e2e through the public API: target H2D from pinned memory + kernel +
    # winners D2H, per step, cold cache
    host_win = torch.empty_like(win, device="cpu").pin_memory()
    e2e = []
    for _ in range(args.steps):
        ap.ap_cache_reset(cache)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(stream)
        tgt.copy_(tgt_host, non_blocking=True)
        ap.ap_collage_run(cache, region, inp, win, stream)
        host_win.copy_(win, non_blocking=True)
        e.record(stream)
        e.synchronize()
        e2e.append(s.elapsed_time(e) * 1e-3)
    cands = None
    res = dict(cfg=cfg, id_chunks=id_chunks, times=times, stats=stats, err=err, got=got, b0=b0, b1=b1, nb=nb,
               fused=fused,
               units=(u0, u1), bucket=bucket, records=bool(i1),
               other=other_res,
               link=link, raw=raw, e2e=e2e, clocks=clk.summary(), t_gen=t_gen, t_pin=t_pin,
               t_index=t_index, h2d=int(tgt_host.numel()), d2h=int(win.numel() * 4),
               is_copy=is_copy, src=src, cands=cands)
    # parity sample vs the oracle (rank 0): all blocks for c4, a sample for c5
    res["parity"] = None
    # the combined answer (N > 1) on rank 0
    full = combine() if world > 1 else None
    if sw is not None:
        sw.close()
    if bucket and rank == 0:
        got = full.cpu().numpy().view(np.uint32).copy()  # rank 0's own array is partial
        res["got"] = got
    po = pi = None
    if rank == 0 and not args.no_cpu_baseline:
        # the oracle's own bucket index (never the GPU-built CSR): the oracle
        # collage runs on it, and the GPU index must equal it
        import oracle
        t0 = time.time()
        po, pi = oracle.build_index(recs, cfg["stride"], cfg["N"], proj, bias, cfg["w"], cfg["bb"],
                                    threads=os.cpu_count() or 1)
        t_oindex = time.time() - t0
        index_equal = bool(np.array_equal(po, off.cpu().numpy().view(np.uint32)) and
                           np.array_equal(pi, ids.cpu().numpy().view(np.uint32)))
    want_all = None
    if rank == 0 and full is not None and not args.no_cpu_baseline:
        # the combined winners of every rank against the oracle, all blocks
        fw = full.cpu().numpy().view(np.uint32)
        want_all = oracle.collage(img, proj, bias, cfg["w"], cfg["bb"], recs, cfg["stride"],
                                  cfg["N"], po, pi, b0=0, nb=nb, threads=os.cpu_count() or 1)
        res["gathered_parity"] = dict(ranks=world, blocks=nb,
                                      equal=bool(np.array_equal(want_all, fw[:nb])),
                                      partition=("records (id slices)" if i1 else "buckets (units)")
                                      if bucket else "blocks")
    if rank == 0 and not args.no_cpu_baseline:
        # rank 0's own blocks, all of them (C5: 65 536 blocks, a few seconds
        # on the host cores), timed as the oracle's collage
        threads = os.cpu_count() or 1
        nsample = b1 - b0
        t0 = time.time()
        want = oracle.collage(img, proj, bias, cfg["w"], cfg["bb"], recs, cfg["stride"], cfg["N"],
                              po, pi, b0=b0, nb=nsample, threads=threads)
        dt = time.time() - t0
        res["parity"] = dict(blocks=nsample, equal=bool(np.array_equal(want, got[:nsample])),
                             cpu_s=dt, cores=threads, index_equal=index_equal,
                             oracle_index_s=round(t_oindex, 2),
                             empty_blocks=int(np.all(want == oracle.EMPTY, axis=1).sum()))
    ap.ap_munmap(cache, region)
    ap.ap_cache_destroy(cache)
    if keep:
        del recs
    return res


def _traffic(kernel):
    try:
        with open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles",
                               "traffic.json")) as f:
            return json.load(f)[kernel]["dram_bytes_per_launch"]
    except Exception:
        return None


def emit_collage(args, res_all, world, METRIC):
    r0 = res_all[0]
    cfg = r0["cfg"]
    tmax = max(sum(r["times"]) for r in res_all) / args.steps
    st = r0["stats"][-1]
    fill = st["fill_bytes"]
    t0 = sum(r0["times"]) / args.steps
    # C5's (window, unit) items run one per warp (k_collage_wunit, >= 2^20 items)
    kname = (f"k_collage_wunit<{args.group}, apointer>" if cfg["name"] == "c5"
             else f"k_collage<{args.group}, apointer>")
    line = {
        "metric": METRIC, "value": round(tmax, 6), "unit": "s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(tmax * 1e3, 3),
        "higher_is_better": False, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
        "data": "synthetic (blob-tile histograms, seeded target with 5% planted copies)",
        "config": {"workload": cfg["workload"], "records": cfg["N"], "target": [cfg["W"], cfg["H"]],
                   "blocks": r0["nb"], "L": cfg["L"], "K": cfg["K"], "bucket_bits": cfg["bb"],
                   "w": cfg["w"], "cache_bytes_per_gpu": cfg["frames"] * cfg["page"],
                   "record_stride": cfg["stride"],
                   "group": args.group,
                   "schedule": SCHED_NAMES[args.schedule],
                   "id_chunks": r0["id_chunks"],
                   "l2": "inputs larger than L2 (multi-GB record file, cold cache per step)",
                   "parallelism": (((f"record-id slices (file shards) over {world} ranks, all units "
                                     "each") if r0.get("records") else
                                    f"(table, bucket) units partitioned over {world} ranks"
                                    if r0.get("bucket") else
                                    f"blocks partitioned over {world} rank(s)") +
                                   ("" if world == 1 else
                                    " + winners folded into rank 0's array by the kernels "
                                    "(CUDA IPC, system-scope atomic min; no collective)"
                                    if r0.get("fused") else
                                    " + NCCL MIN reduce" if r0.get("bucket") else
                                    " + NCCL gather"))},
        "collage": {"blocks_rank0": r0["b1"] - r0["b0"],
                    "units_rank0": (r0["units"][1] - r0["units"][0]) if r0.get("bucket") else None,
                    "major_faults": st["major"],
                    "minor_faults": st["minor"], "evictions": st["evictions"],
                    "fill_GB": round(fill / 1e9, 3), "waits": st["waits"],
                    "device_error": r0["err"], "setup_s": {"generate": round(r0["t_gen"], 2),
                                                          "pin": round(r0["t_pin"], 2),
                                                          "index_build_gpu": round(r0["t_index"], 3)},
                    "per_rank_s": [round(sum(r["times"]) / args.steps, 6) for r in res_all],
                    "other_schedules": [{k: (round(v, 6) if isinstance(v, float) else v)
                                         for k, v in o.items()} for o in r0["other"]]},
        "roofline": {"bound": "host_link", "achieved": round(fill / t0 / 1e9, 3),
                     "peak": round(r0["link"], 3), "unit": "GB/s",
                     "frac": round(fill / t0 / 1e9 / r0["link"], 4),
                     "traffic": _traffic(kname),
                     "traffic_note": "DRAM bytes of one step = one launch (the record-id windows "
                                     "are fused), from the committed ncu --set full capture "
                                     "(profiles/traffic.json)",
                     "algorithmic_bytes_per_step": int(fill),
                     "kernel": kname,
                     "peak_source": "host->device cudaMemcpy from pinned memory, this run"},
        "e2e": {"value": round(max(np.mean(r["e2e"]) for r in res_all), 6), "unit": "s",
                "h2d_bytes_per_step": r0["h2d"], "d2h_bytes_per_step": r0["d2h"],
                "api": "target H2D + ap_collage_run + winners D2H (cold cache)"},
        "gpu_launches": args.steps * ((2 + max(1, r0["id_chunks"])) if args.schedule else 1),
        "gpu_launches_note": "per step: k_collage once per record-id window (id_chunks), plus "
                             "k_collage_keys and k_iota32 for the sorted schedules; the "
                             "schedule's radix sort adds cub library kernels",
        "clocks": r0["clocks"],
    }
    if r0["raw"]:
        line["collage"]["raw_twin_resident_hbm_s"] = round(r0["raw"]["raw_s"], 6)
        line["collage"]["apointer_warm_cache_s"] = round(r0["raw"]["warm_s"], 6)
        line["collage"]["overhead_warm_vs_raw"] = round(r0["raw"]["warm_s"] / r0["raw"]["raw_s"] - 1, 4)
        line["collage"]["raw_twin_equal"] = r0["raw"]["equal"]
        if "resident" in r0["raw"]:
            line["collage"]["resident_cache"] = {
                f"group{g}": {k: (round(v, 6) if isinstance(v, float) else v) for k, v in d.items()}
                for g, d in r0["raw"]["resident"].items()}
            line["collage"]["resident_cache"]["note"] = (
                "cache holds every record (prefilled): apointer collage vs the identical kernel on "
                "a raw pointer into an HBM copy; majors after prefill: "
                f"{r0['raw']['resident_majors']}")
    if r0.get("gathered_parity"):
        line["collage"]["gathered_parity_vs_oracle"] = r0["gathered_parity"]
    if r0["parity"]:
        p = r0["parity"]
        line["collage"]["parity_vs_oracle"] = {k: v for k, v in p.items() if k != "cpu_s"}
        full_blocks = r0["b1"] - r0["b0"]
        line["cpu_baseline"] = {"value": round(p["cpu_s"] * full_blocks / p["blocks"], 4),
                                "unit": "s", "cores": p["cores"], "kind": "oracle",
                                "sample": (f"oracle collage over all {full_blocks} of rank 0's "
                                           "blocks on its own bucket index (index build "
                                           "excluded)") if p["blocks"] == full_blocks else
                                          (f"oracle collage over {p['blocks']} of rank 0's "
                                           f"{full_blocks} blocks, scaled to all of them")}
    return line


def collage_summary(args, res_all, world):
    """The C4 collage object embedded in the default bench line (BASELINE.json
    configs[3]): seconds per cold step (max over ranks),
    its spread, fills, the host-link bound of the distinct records, the
    resident-cache apointer vs raw-twin overhead, parity and the oracle."""
    r0 = res_all[0]
    cfg = r0["cfg"]
    per_rank = [float(np.mean(r["times"])) for r in res_all]
    tmax = max(per_rank)
    st = r0["stats"][-1]
    t = np.asarray(r0["times"]) * 1e3
    out = {
        "workload": cfg["workload"], "schedule": SCHED_NAMES[args.schedule],
        "group": args.group, "id_chunks": r0["id_chunks"],
        "parallelism": ("record-id slices over %d ranks" % world) if r0.get("records") else
                       ("units over %d ranks" % world) if r0.get("bucket") else
                       ("blocks over %d rank(s)" % world),
        "s": round(tmax, 6), "per_rank_s": [round(x, 6) for x in per_rank],
        "step_times": {"mean_ms": round(float(t.mean()), 4),
                       "std_ms": round(float(t.std(ddof=1)) if len(t) > 1 else 0.0, 4),
                       "n": int(len(t))},
        "fill_GB": round(st["fill_bytes"] / 1e9, 4), "major_faults": st["major"],
        "device_error": r0["err"], "host_link_GBps": round(r0["link"], 2),
        "fill_frac_of_host_link": round(st["fill_bytes"] / float(np.mean(r0["times"])) / 1e9 /
                                        r0["link"], 4),
        "e2e_s": round(max(float(np.mean(r["e2e"])) for r in res_all), 6),
        "setup_s": {"generate": round(r0["t_gen"], 2), "pin": round(r0["t_pin"], 2),
                    "index": round(r0["t_index"], 3)},
    }
    # the collage kernel is fill-bound: its roofline is the host link (page
    # fill bytes per second of the device-timed step, one launch per step)
    fill_rate = st["fill_bytes"] / float(np.mean(r0["times"])) / 1e9
    # C5's 25 M (window, unit) items run one per warp (k_collage_wunit)
    kname = "k_collage_wunit<8, apointer>" if cfg["name"] == "c5" else "k_collage<8, apointer>"
    if cfg["name"] == "c5":
        out["traffic_note"] = ("ncu DRAM bytes per launch (profiles/r02_full_c5.txt): 87 GB of reads are "
                               "the candidates' payload re-read from the frames (~120 GB of record "
                               "reads, L2 serves the rest) and 51 GB of writes = 24 GB of fills + the "
                               "rest, L2 evictions of local-memory (spill) lines of the fault path "
                               "(8.2 G local store sectors per launch, 3.6 G of them L1 misses); HBM "
                               "runs at 0.28 TB/s, the host link is the bound")
    from bench import ncu_traffic
    out["roofline"] = {"bound": "host_link", "achieved": round(fill_rate, 3),
                       "peak": round(r0["link"], 3), "unit": "GB/s",
                       "frac": round(fill_rate / r0["link"], 4),
                       "traffic": ncu_traffic(kname),
                       "algorithmic_bytes_per_launch": int(st["fill_bytes"]),
                       "kernel": kname + " (the step's record-id windows fused in one launch)",
                       "peak_source": "host->device cudaMemcpy from pinned memory, this run"}
    raw = r0.get("raw")
    if raw:
        bound = raw["distinct_pages"] * cfg["page"] / (r0["link"] * 1e9)
        out["distinct_record_pages"] = raw["distinct_pages"]
        out["distinct_bound_s"] = round(bound, 6)
        out["frac_of_distinct_bound"] = round(bound / float(np.mean(r0["times"])), 4)
        out["resident"] = {f"group{g}": {"apointer_ms": round(d["apointer_s"] * 1e3, 4),
                                         "raw_ms": round(d["raw_s"] * 1e3, 4),
                                         "overhead": round(d["overhead"], 4), "equal": d["equal"]}
                           for g, d in raw["resident"].items()}
    if r0.get("parity"):
        p = r0["parity"]
        out["parity_vs_oracle"] = {k: v for k, v in p.items() if k not in ("cpu_s",)}
        full_blocks = r0["b1"] - r0["b0"]
        out["oracle_s"] = round(p["cpu_s"] * full_blocks / p["blocks"], 4)
        out["oracle_cores"] = p["cores"]
        if p["blocks"] < full_blocks:
            out["oracle_s_note"] = (f"the oracle ran {p['blocks']} of {full_blocks} blocks; "
                                    "oracle_s scales its time to all blocks")
    if r0.get("gathered_parity"):
        out["gathered_parity_vs_oracle"] = r0["gathered_parity"]
    return out
