"""Read workloads C1 and C3 for bench.py (--workload c1 | c3).

C1 (BASELINE configs[0]): 16 MB file, 4 KB pages, 64-frame cache, one warp
per SM reading sequentially (148 warps contend for 64 frames: every page is a
major fault and most fills evict).  Output = the whole file copied through
apointers, compared byte for byte with the file.
C3 (configs[2]): divergent-warp stress -- each of the 32 lanes of a warp on a
distinct page, 256 MiB cache over a 16 GiB file, 4 KiB pages (DESIGN.md
R-A10), 4-B reads, all SMs.  Output = per-thread checksums vs the oracle.
A step = cold cache (reset, untimed) + one kernel launch, CUDA-event timed.
"""
import os
import time

import numpy as np

GiB = 1 << 30


def read_config(name, reads):
    if name == "c1":
        return dict(name="c1", file_bytes=16 << 20, page=4096, frames=64, grid=148, block=32,
                    pattern="seq", elem=16, unit=4096,
                    workload="C1: 16 MiB file, 4 KiB pages, 64-frame cache, 1 warp/SM "
                             "sequential 16-B apointer reads (page units from a work queue), "
                             "full copy out, cold per step")
    return dict(name="c3", file_bytes=16 * GiB, page=4096, frames=65536, grid=148, block=512,
                pattern="divergent", elem=4, reads=max(reads // 2, 1),
                workload="C3: divergent-warp stress, 32 lanes on 32 distinct 4 KiB pages, 256 MiB "
                         "cache over a 16 GiB file, 4-B apointer reads, all SMs, cold per step")


def run_reads(args, torch, dev, rank, world, dist, timed, ClockSampler, host_link_peak,
              aligned_empty):
    import paper_conf_isca_shaharbs16_b200 as ap
    import synth
    cfg = read_config(args.workload, args.reads)
    stream = torch.cuda.current_stream()
    f = synth.fill_file(aligned_empty(cfg["file_bytes"]), 1 + rank)
    cache = ap.ap_cache_create(cfg["frames"], cfg["page"], torch.cuda.current_device())
    region = ap.ap_mmap(cache, f)
    nthreads = cfg["grid"] * cfg["block"]
    rr = None
    if cfg["pattern"] == "seq":
        out = torch.empty(cfg["file_bytes"], dtype=torch.uint8, device=dev)
        # units from a work queue (AP_SEQ_QUEUE): with 148 warps over 64
        # frames, round robin (AP_SEQ, measured beside it) leaves the last
        # warps streaming alone while most frames sit idle
        bc = ap.bench_cfg(ap.AP_SEQ_QUEUE, cfg["elem"], cfg["grid"], cfg["block"],
                          unit_bytes=cfg["unit"], out_copy=True)
        rr = ap.bench_cfg(ap.AP_SEQ, cfg["elem"], cfg["grid"], cfg["block"],
                          unit_bytes=cfg["unit"], out_copy=True)
        raw = ap.bench_cfg(ap.AP_SEQ_QUEUE, cfg["elem"], cfg["grid"], cfg["block"],
                           unit_bytes=cfg["unit"], out_copy=True, mode=ap.AP_MODE_RAW,
                           raw_base=ap.ap_region_devptr(cache, region))
        reads = cfg["file_bytes"] // cfg["elem"]
    else:
        out = torch.empty(nthreads, dtype=torch.int64, device=dev)
        bc = ap.bench_cfg(ap.AP_DIVERGENT, cfg["elem"], cfg["grid"], cfg["block"],
                          reads_per_thread=cfg["reads"], page_bytes=cfg["page"], seed=77)
        raw = ap.bench_cfg(ap.AP_DIVERGENT, cfg["elem"], cfg["grid"], cfg["block"],
                           reads_per_thread=cfg["reads"], page_bytes=cfg["page"], seed=77,
                           mode=ap.AP_MODE_RAW, raw_base=ap.ap_region_devptr(cache, region))
        reads = nthreads * cfg["reads"]
    # eviction policy: C1 is a single-pass stream, so the drop-behind hint
    # (AP_POLICY_SEQUENTIAL) by default; the clock alone is measured beside it
    pol_names = {"clock": ap.AP_POLICY_CLOCK, "sequential": ap.AP_POLICY_SEQUENTIAL}
    policy = args.policy or ("sequential" if cfg["name"] == "c1" else "clock")
    ap.ap_cache_set_policy(cache, pol_names[policy])
    cfg["policy"] = policy
    link = host_link_peak(torch, dev)
    step = lambda: ap.ap_bench_read(cache, region, bc, out, stream)  # noqa: E731
    for _ in range(args.warmup):
        ap.ap_cache_reset(cache)
        timed(torch, step, stream)
    times, stats = [], []
    with ClockSampler(torch.cuda.current_device()) as clk:
        for _ in range(args.steps):
            ap.ap_cache_reset(cache)
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            times.append(timed(torch, step, stream))
            stats.append(ap.ap_cache_stats(cache))
    err = ap.ap_last_device_error(cache)
    got = out.cpu().numpy()
    other = {}
    for name, pol in pol_names.items():
        if name == policy:
            continue
        ap.ap_cache_set_policy(cache, pol)
        out_o = torch.empty_like(out)
        to = []
        for _ in range(3):
            ap.ap_cache_reset(cache)
            to.append(timed(torch, lambda: ap.ap_bench_read(cache, region, bc, out_o, stream),
                            stream))
        so = ap.ap_cache_stats(cache)
        other[name] = dict(s=min(to), fill_GBps=so["fill_bytes"] / min(to) / 1e9,
                           evictions=so["evictions"], equal=bool(torch.equal(out_o, out)))
        ap.ap_cache_set_policy(cache, pol_names[policy])
    if rr is not None:
        out_o = torch.empty_like(out)
        to = []
        for _ in range(3):
            ap.ap_cache_reset(cache)
            to.append(timed(torch, lambda: ap.ap_bench_read(cache, region, rr, out_o, stream),
                            stream))
        so = ap.ap_cache_stats(cache)
        other["round_robin_units"] = dict(s=min(to), fill_GBps=so["fill_bytes"] / min(to) / 1e9,
                                          evictions=so["evictions"],
                                          equal=bool(torch.equal(out_o, out)))
    out_raw = torch.empty_like(out)
    raw_t = min(timed(torch, lambda: ap.ap_bench_read(cache, region, raw, out_raw, stream), stream)
                for _ in range(3))
    raw_equal = bool(torch.equal(out_raw, out))
    # parity vs the oracle (rank 0)
    parity = None
    if rank == 0 and not args.no_cpu_baseline:
        import oracle
        threads = os.cpu_count() or 1
        t0 = time.time()
        if cfg["pattern"] == "seq":
            want = oracle.read_seq(f, cfg["file_bytes"], cfg["unit"], cfg["elem"], nthreads, 1,
                                   copy=True, threads=threads)
            eq = bool(np.array_equal(want, got)) and bool(np.array_equal(got, f))
        else:
            want = oracle.read_divergent(f, cfg["file_bytes"], cfg["page"], cfg["elem"], nthreads,
                                         cfg["reads"], 77, threads=threads)
            eq = bool(np.array_equal(want, got.view(np.uint64)))
        parity = dict(equal=eq, cpu_s=time.time() - t0, cores=threads)
    ap.ap_munmap(cache, region)
    ap.ap_cache_destroy(cache)
    return dict(cfg=cfg, times=times, stats=stats, err=err, link=link, raw_t=raw_t,
                raw_equal=raw_equal, reads=reads, clocks=clk.summary(), parity=parity,
                other_policies=other)


def _traffic(kernel):
    """DRAM bytes per launch of `kernel` from the committed ncu capture
    (profiles/traffic.json), or None."""
    import json
    try:
        with open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles",
                               "traffic.json")) as f:
            return json.load(f)[kernel]["dram_bytes_per_launch"]
    except Exception:
        return None


def emit_reads(args, res_all, world, METRIC):
    r0 = res_all[0]
    cfg = r0["cfg"]
    tmax = max(sum(r["times"]) for r in res_all) / args.steps
    fill_all = sum(r["stats"][-1]["fill_bytes"] for r in res_all)
    st = r0["stats"][-1]
    t0 = sum(r0["times"]) / args.steps
    line = {
        "metric": METRIC, "value": round(fill_all / tmax / 1e9, 3), "unit": "GB/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(tmax * 1e3, 3), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32" if cfg["elem"] == 4 else "u128",
        "data": "synthetic (splitmix64 file words)",
        "config": {"workload": cfg["workload"], "file_bytes": cfg["file_bytes"],
                   "page_bytes": cfg["page"], "frames": cfg["frames"], "grid": cfg["grid"],
                   "block": cfg["block"], "reads_per_step": r0["reads"],
                   "eviction_policy": cfg["policy"],
                   "l2": "cold cache per step; file > L2" if cfg["name"] == "c3" else
                         "cold cache per step (16 MiB file fits L2: C1 measures the fault path)",
                   "parallelism": f"replicas x{world}"},
        "fault_bound": {"fill_GBps": round(st["fill_bytes"] / t0 / 1e9, 3),
                        "host_link_GBps_memcpy": round(r0["link"], 2),
                        "frac_of_host_link": round(st["fill_bytes"] / t0 / 1e9 / r0["link"], 4),
                        "reads_per_s": round(r0["reads"] / t0, 1),
                        "major_faults": st["major"], "minor_faults": st["minor"],
                        "evictions": st["evictions"], "waits": st["waits"],
                        "downgrades": st["downgrades"], "nofree": st["nofree"],
                        "raw_zero_copy_twin_s": round(r0["raw_t"], 6),
                        "raw_twin_equal": r0["raw_equal"], "device_error": r0["err"],
                        "other_policies": {k: {kk: (round(vv, 6) if isinstance(vv, float) else vv)
                                               for kk, vv in v.items()}
                                           for k, v in r0.get("other_policies", {}).items()}},
        "roofline": {"bound": "host_link", "achieved": round(st["fill_bytes"] / t0 / 1e9, 3),
                     "peak": round(r0["link"], 3), "unit": "GB/s",
                     "frac": round(st["fill_bytes"] / t0 / 1e9 / r0["link"], 4),
                     "traffic": _traffic("k_seq_queue<uint4, apointer>" if cfg["name"] == "c1"
                                         else "k_random<uint32_t, DIVERGENT, apointer>"),
                     "kernel": ("k_seq_queue<uint4, apointer>" if cfg["name"] == "c1"
                                else "k_random<uint32_t, DIVERGENT, apointer>"),
                     "algorithmic_bytes_per_launch": int(st["fill_bytes"]),
                     "peak_source": "host->device cudaMemcpy from pinned memory, this run"},
        "gpu_launches": args.steps, "clocks": r0["clocks"],
    }
    if r0["parity"]:
        line["parity_vs_oracle"] = {k: v for k, v in r0["parity"].items() if k != "cpu_s"}
        line["cpu_baseline"] = {"value": round(r0["reads"] * cfg["elem"] / r0["parity"]["cpu_s"]
                                               / 1e9, 6), "unit": "GB/s",
                                "cores": r0["parity"]["cores"], "kind": "oracle",
                                "sample": "the whole read set, plain file indexing; bytes read / s"}
    return line


def reads_summary(args, res_all, world, METRIC):
    """The C1 / C3 line (emit_reads) as a sub-object of the default line: the
    driver then runs these configs too (cold cache per step, device-timed,
    parity vs the oracle on rank 0)."""
    line = emit_reads(args, res_all, world, METRIC)
    times = [t for r in res_all for t in r["times"]]
    mean = sum(times) / len(times)
    std = (sum((t - mean) ** 2 for t in times) / max(len(times) - 1, 1)) ** 0.5
    keep = ("value", "unit", "ms_per_step", "dtype", "config", "fault_bound", "roofline",
            "parity_vs_oracle", "cpu_baseline", "clocks")
    out = {k: line[k] for k in keep if k in line}
    out["value_note"] = "page-fill bytes per second over the host link (the fault path's rate)"
    out["step_times"] = {"mean_ms": round(mean * 1e3, 4), "std_ms": round(std * 1e3, 4),
                         "n": len(times)}
    return out
