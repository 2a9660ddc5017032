#!/usr/bin/env python
"""bench.py -- apointer read throughput on B200 (BASELINE.json metric).

Default workload = BASELINE.json configs[1] (C2): a 4 GiB synthetic file in
pinned host memory, 64 KiB pages, a 1 GiB page cache in HBM, uniform-random
4-byte apointer reads from every SM, starting from a cold cache each step
("the first execution ... major page faults").  One step = one
launch of the apointer read kernel over the whole read set; every step runs
the whole hot path (S1-S10 of SURVEY.md §8(a)): translation, warp
aggregation, minor/major faults, clock eviction, host-link fills, publish,
unlink.

`value` = apointer read throughput in USEFUL bytes: 4 B per read returned
to the threads, per second of the device-timed step -- the same quantity the
reference arm (the CPU oracle reading the file directly) prints, so the
driver's ratio compares the same work.  The fault path's own throughput --
the 64 KiB page fills it pulls over the host link per second, against the
host link measured in the same run -- is the roofline object (SURVEY.md
§8(d) M2).  The same JSON line also carries the cache-hit mode (HBM-bound, vs
the raw-pointer twin), the minor-fault regime, the raw zero-copy twin of C2,
and the C4 photo collage (BASELINE.json configs[3]).

Other workloads: --workload c1 | c3 | c4 | c5.
`--impl reference` times the CPU oracle (oracle/) on the host cores instead.
"""
import argparse
import json
import os
import subprocess
import sys
import tempfile
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

GiB = 1 << 30
METRIC = "apointer read GB/s (hit and fault-bound) vs raw ptr; collage s at 1/2/4/8 B200"


def env_rank():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("LOCAL_RANK", 0)),
            int(os.environ.get("WORLD_SIZE", 1)))


# NUMA node of this rank's GPU (main() puts it in AP_BENCH_NODE): host
# "files" the bench creates are bound to it before their first touch, so the
# fault path's zero-copy fills read the socket the GPU's PCIe link hangs off
# (AP_NUMA_LOCAL=0: off)


def gpu_numa_node(torch, dev):
    """The host NUMA node of `dev` from sysfs (None if unknown)."""
    try:
        pr = torch.cuda.get_device_properties(dev)
        bus = f"{pr.pci_domain_id:04x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
        with open(f"/sys/bus/pci/devices/{bus}/numa_node") as f:
            n = int(f.read().strip())
        return n if n >= 0 else None
    except Exception:
        return None


def numa_bind(arr, node):
    """mbind(MPOL_BIND) the pages of a not-yet-touched host buffer to `node`."""
    import ctypes
    libc = ctypes.CDLL(None, use_errno=True)
    page = 4096
    addr = arr.ctypes.data & ~(page - 1)
    length = arr.ctypes.data + arr.nbytes - addr
    nm = ctypes.c_ulong(1 << node)
    SYS_mbind, MPOL_BIND = 237, 2  # x86_64
    return libc.syscall(SYS_mbind, ctypes.c_void_p(addr), ctypes.c_ulong(length), MPOL_BIND,
                        ctypes.byref(nm), ctypes.c_ulong(node + 2), 0) == 0


def aligned_empty(nbytes, align=1 << 21):
    raw = np.empty(nbytes + align, dtype=np.uint8)
    off = (-raw.ctypes.data) % align
    arr = raw[off:off + nbytes]
    node = os.environ.get("AP_BENCH_NODE")  # set by main() (other modules import bench anew)
    if node:
        numa_bind(arr, int(node))
    return arr


def ncu_traffic(kernel):
    """dram read+write bytes per launch of `kernel` from the committed ncu
    capture (profiles/traffic.json), or None."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            return json.load(f)[kernel]["dram_bytes_per_launch"]
    except Exception:
        return None


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured (MEASURED_PEAKS.json)"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.path = tempfile.mktemp(suffix=".csv")

    def __enter__(self):
        try:
            self.f = open(self.path, "w")
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}",
                                          f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "100"], stdout=self.f,
                                         stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            self.proc.wait()
            self.f.close()

    def summary(self):
        rows = []
        try:
            for line in open(self.path):
                p = [x.strip() for x in line.split(",")]
                if len(p) >= 9:
                    rows.append(p)
        except Exception:
            pass
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = sorted(float(r[1]) for r in rows)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({n for r in rows for n, v in zip(names, r[5:9]) if v == "Active"})
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": float(rows[0][2]),
                "samples": len(rows), "reasons": reasons}


# ------------------------------------------------------------------ workloads
def c2_config(args):
    return dict(workload="C2: 4 GiB file in pinned host memory, 64 KiB pages, 1 GiB page cache, "
                         "uniform-random 4-B apointer reads from all SMs, cold cache per step",
                file_bytes=4 * GiB, page=65536, frames=16384, grid=148, block=512,
                reads_per_thread=args.reads, elem=4, seed=1234, file_seed=1)


def host_link_peak(torch, dev):
    """Host->device bandwidth measured in this run: cudaMemcpy from pinned
    memory (copy engine), best of 5 x 1 GiB."""
    h = torch.empty(GiB, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(GiB, dtype=torch.uint8, device=dev)
    best = 0.0
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for _ in range(6):
        s.record()
        d.copy_(h, non_blocking=True)
        e.record()
        e.synchronize()
        best = max(best, GiB / (s.elapsed_time(e) * 1e-3) / 1e9)
    del h, d
    return best


def timed(torch, fn, stream):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record(stream)
    fn()
    e.record(stream)
    e.synchronize()
    return s.elapsed_time(e) * 1e-3


def run_c2(args, torch, dev, rank, world, dist):
    import paper_conf_isca_shaharbs16_b200 as ap
    import synth
    cfgd = c2_config(args)
    stream = torch.cuda.current_stream()
    t_setup = time.time()
    f = synth.fill_file(aligned_empty(cfgd["file_bytes"]), cfgd["file_seed"] + rank)
    cache = ap.ap_cache_create(cfgd["frames"], cfgd["page"], torch.cuda.current_device())
    region = ap.ap_mmap(cache, f)
    t_setup = time.time() - t_setup
    nthreads = cfgd["grid"] * cfgd["block"]
    out = torch.empty(nthreads, dtype=torch.int64, device=dev)
    cfg = ap.bench_cfg(ap.AP_UNIFORM, cfgd["elem"], cfgd["grid"], cfgd["block"],
                       reads_per_thread=cfgd["reads_per_thread"], seed=cfgd["seed"])
    link = host_link_peak(torch, dev)

    def step():
        ap.ap_bench_read(cache, region, cfg, out, stream)

    for _ in range(args.warmup):
        ap.ap_cache_reset(cache)
        timed(torch, step, stream)
    times, fills, stats = [], [], []
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(torch.cuda.current_device()) as clk:
        for _ in range(args.steps):
            ap.ap_cache_reset(cache)  # cold start each step (untimed)
            times.append(timed(torch, step, stream))
            st = ap.ap_cache_stats(cache)
            stats.append(st)
            fills.append(st["fill_bytes"])
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    err = ap.ap_last_device_error(cache)
    total_t = sum(times)
    total_fill = sum(fills)
    # parity of the last step against the oracle is done by tests; here we
    # keep the checksums for the cpu_baseline comparison (rank 0, N=1)
    got = out.cpu().numpy().view(np.uint64)

    # raw zero-copy twin: identical kernel on the host alias (no page cache)
    base = ap.ap_region_devptr(cache, region)
    cfg_raw = ap.bench_cfg(ap.AP_UNIFORM, cfgd["elem"], cfgd["grid"], cfgd["block"],
                           reads_per_thread=cfgd["reads_per_thread"], seed=cfgd["seed"],
                           mode=ap.AP_MODE_RAW, raw_base=base)
    out_raw = torch.empty_like(out)
    raw_t = min(timed(torch, lambda: ap.ap_bench_read(cache, region, cfg_raw, out_raw, stream),
                      stream) for _ in range(3))
    raw_match = bool(torch.equal(out_raw, out))
    # zero-copy bulk read of 1 GiB through SMs (SEQ raw over the host alias)
    cfg_zc = ap.bench_cfg(ap.AP_SEQ, 16, 148 * 4, 512, unit_bytes=16384, passes=1,
                          span_bytes=GiB, mode=ap.AP_MODE_RAW, raw_base=base)
    zc_out = torch.empty(148 * 4 * 512, dtype=torch.int64, device=dev)
    zc_t = min(timed(torch, lambda: ap.ap_bench_read(cache, region, cfg_zc, zc_out, stream),
                     stream) for _ in range(3))
    zc_gbs = GiB / zc_t / 1e9

    # e2e: the C-ABI call with a host output buffer (launch + D2H of checksums)
    host_out = torch.empty(nthreads, dtype=torch.int64, pin_memory=True)
    e2e_t, e2e_fill = [], 0
    for _ in range(args.steps):
        ap.ap_cache_reset(cache)
        e2e_t.append(ap.ap_bench_read_host(cache, region, cfg, host_out.numpy()))
        e2e_fill += ap.ap_cache_stats(cache)["fill_bytes"]
    e2e_match = bool(np.array_equal(host_out.numpy().view(np.uint64), out.cpu().numpy().view(np.uint64)))

    # cache-hit mode (M2h): warm the first 1 GiB, stream it 8x with 16-B reads
    hit = run_hit(args, torch, dev, ap, cache, region, f, stream)

    reads = nthreads * cfgd["reads_per_thread"]
    res = dict(cfgd=cfgd, times=times, total_t=total_t, total_fill=total_fill, stats=stats,
               err=err, link=link, zc_gbs=zc_gbs, raw_t=raw_t, raw_match=raw_match,
               reads=reads, e2e_t=e2e_t, e2e_fill=e2e_fill, e2e_match=e2e_match, hit=hit, setup_s=t_setup,
               clocks=clk.summary(), got=got, file=f, nthreads=nthreads)
    ap.ap_munmap(cache, region)
    ap.ap_cache_destroy(cache)
    return res


def run_hit(args, torch, dev, ap, cache, region, f, stream, span=GiB, passes=8):
    """Cache-hit mode: the first 1 GiB is made resident,
    then every warp walks whole 64 KiB pages with 16-B reads, 8 passes.
    Three apointer access styles against the identical kernel
    on a raw pointer into an HBM copy of the same bytes."""
    page = 65536
    ap.ap_cache_reset(cache)
    ap.ap_prefill(cache, region, 0, span // page, stream)
    torch.cuda.synchronize()
    st0 = ap.ap_cache_stats(cache)
    grid, block = 148, 512
    nthreads = grid * block
    out = torch.empty(nthreads, dtype=torch.int64, device=dev)
    dcopy = torch.from_numpy(f[:span]).to(dev)
    out_raw = torch.empty_like(out)
    cfg_raw = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=page, passes=passes,
                           span_bytes=span, mode=ap.AP_MODE_RAW, raw_base=dcopy.data_ptr())
    nbytes = span * passes

    def run(cfg, o):
        for _ in range(max(args.warmup, 3)):
            ap.ap_bench_read(cache, region, cfg, o, stream)
        return [timed(torch, lambda: ap.ap_bench_read(cache, region, cfg, o, stream), stream)
                for _ in range(max(args.steps, 5))]

    def paired(cfg, o, n):
        """apointer and raw twin launched alternately (launch by launch), so
        clock or thermal drift during the run cannot favour either side"""
        for _ in range(max(args.warmup, 3)):
            ap.ap_bench_read(cache, region, cfg, o, stream)
            ap.ap_bench_read(cache, region, cfg_raw, out_raw, stream)
        ta, tr = [], []
        for _ in range(n):
            ta.append(timed(torch, lambda: ap.ap_bench_read(cache, region, cfg, o, stream), stream))
            tr.append(timed(torch, lambda: ap.ap_bench_read(cache, region, cfg_raw, out_raw, stream),
                            stream))
        return np.array(ta), np.array(tr)

    n_pairs = max(args.steps, 10)
    res = dict(bytes_per_launch=nbytes, pairs=n_pairs)
    same = True
    t_raw_all = []
    for acc, name in ((ap.AP_ACCESS_TILE, "tile"), (ap.AP_ACCESS_RANGE, "range")):
        cfg = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=page, passes=passes,
                           span_bytes=span, access=acc)
        t, tr = paired(cfg, out, n_pairs)
        t_raw_all.extend(tr)
        same = same and bool(torch.equal(out, out_raw))
        res[name] = dict(s=float(np.mean(t)), gbs=nbytes / np.mean(t) / 1e9,
                         raw_gbs=nbytes / np.mean(tr) / 1e9,
                         overhead=float(np.median(t / tr) - 1),
                         overhead_of_means=float(np.mean(t) / np.mean(tr) - 1))
    t_raw = np.array(t_raw_all)
    res.update(raw_s=float(np.mean(t_raw)), raw_gbs=nbytes / np.mean(t_raw) / 1e9)
    # per-access form: `v = *q; q += 32`, AP_DEREF_PIPE dereferences in
    # flight per lane, one CTA of 512 per SM (the kernel's launch bounds);
    # its twin is the same per-access loop on a raw pointer at the same launch
    grid_d = 148
    out_d = torch.empty(grid_d * block, dtype=torch.int64, device=dev)
    out_rd = torch.empty_like(out_d)
    cfg_rd = ap.bench_cfg(ap.AP_SEQ, 16, grid_d, block, unit_bytes=page, passes=passes,
                          span_bytes=span, mode=ap.AP_MODE_RAW, raw_base=dcopy.data_ptr(),
                          access=ap.AP_ACCESS_DEREF)
    cfg_d = ap.bench_cfg(ap.AP_SEQ, 16, grid_d, block, unit_bytes=page, passes=passes,
                         span_bytes=span, access=ap.AP_ACCESS_DEREF)
    t_rd = run(cfg_rd, out_rd)
    t = run(cfg_d, out_d)
    same = same and bool(torch.equal(out_d, out_rd))
    res["deref"] = dict(s=float(np.mean(t)), gbs=nbytes / np.mean(t) / 1e9,
                        overhead=float(np.mean(t) / np.mean(t_raw) - 1),
                        raw_deref_gbs=nbytes / np.mean(t_rd) / 1e9,
                        overhead_vs_raw_deref=float(np.mean(t) / np.mean(t_rd) - 1), grid=grid_d)
    st1 = ap.ap_cache_stats(cache)
    # M2r: uniform-random 4-B reads over the resident GiB, so
    # every read leaves its page: an unlink + a minor fault per read, vs the
    # raw gather from the HBM copy.  Full occupancy for both (one read in
    # flight per thread between faults).
    grid_m, reads_m = 4 * 148, 8
    out_m = torch.empty(grid_m * block, dtype=torch.int64, device=dev)
    out_mr = torch.empty_like(out_m)
    cfg_m = ap.bench_cfg(ap.AP_UNIFORM, 4, grid_m, block, reads_per_thread=reads_m, seed=11,
                         span_bytes=span)
    cfg_mr = ap.bench_cfg(ap.AP_UNIFORM, 4, grid_m, block, reads_per_thread=reads_m, seed=11,
                          span_bytes=span, mode=ap.AP_MODE_RAW, raw_base=dcopy.data_ptr())
    st_m0 = ap.ap_cache_stats(cache)
    t_m = run(cfg_m, out_m)
    st_m1 = ap.ap_cache_stats(cache)
    t_mr = run(cfg_mr, out_mr)
    nreads = grid_m * block * reads_m
    res["minor"] = dict(
        reads_per_launch=nreads, s=float(np.mean(t_m)), raw_s=float(np.mean(t_mr)),
        reads_per_s=nreads / np.mean(t_m), raw_reads_per_s=nreads / np.mean(t_mr),
        useful_gbs=4 * nreads / np.mean(t_m) / 1e9, sector_gbs=32 * nreads / np.mean(t_m) / 1e9,
        overhead=float(np.mean(t_m) / np.mean(t_mr) - 1),
        majors=st_m1["major"] - st_m0["major"],
        minors_per_launch=(st_m1["minor"] - st_m0["minor"]) / max(1, len(t_m) + max(args.warmup, 3)),
        equal_raw=bool(torch.equal(out_m, out_mr)), grid=grid_m)
    # the M2r ceiling, measured here: the same memory operations per read (an
    # acquire add and a release add on random entries of a 16 384-entry PTE
    # array + the 4-B gather) with no page-cache logic (tools/atomic_ceiling.cu)
    res["minor"]["ceiling"] = m2r_ceiling()
    del dcopy
    res.update(majors_during=st1["major"] - st0["major"], checksums_equal_raw=same,
               ap_gbs=res["tile"]["gbs"], overhead=res["tile"]["overhead"])
    return res


def m2r_ceiling():
    """G steps/s of tools/atomic_ceiling (built by make), or None."""
    exe = os.path.join(ROOT, "tools", "atomic_ceiling")
    if not os.path.exists(exe):
        return None
    try:
        out = subprocess.run([exe], capture_output=True, text=True, timeout=120).stdout
    except Exception:
        return None
    import re
    res = {}
    for line in out.splitlines():
        m = re.match(r"^(.*?)\s+([0-9.]+) G steps/s", line)
        if m:
            res[m.group(1).strip()] = float(m.group(2)) * 1e9
    return res or None


def cpu_oracle_c2(res, threads):
    """The oracle as it stands (plain file indexing + FNV), on the host cores:
    first the bench's own read set (checked against the GPU checksums), then
    fresh seeds (so no pass re-reads lines a previous pass left in the CPU
    caches) until >= 3 s of CPU work."""
    import oracle
    cfgd = res["cfgd"]
    f = res["file"]
    ck = oracle.read_uniform(f, cfgd["file_bytes"], cfgd["elem"], res["nthreads"],
                             cfgd["reads_per_thread"], cfgd["seed"], threads=threads)
    match = bool(np.array_equal(ck, res["got"]))
    t0 = time.time()
    n = 0
    while time.time() - t0 < 3.0:
        oracle.read_uniform(f, cfgd["file_bytes"], cfgd["elem"], res["nthreads"],
                            cfgd["reads_per_thread"], cfgd["seed"] + 1000 + n, threads=threads)
        n += 1
    dt = (time.time() - t0) / n
    return dt, match, n


def step_stats(times):
    """Mean and spread of the timed steps (the paper reports the mean of its
    last 7 of 10 runs with the standard deviation)."""
    t = np.asarray(times, dtype=np.float64) * 1e3
    return {"mean_ms": round(float(t.mean()), 4), "std_ms": round(float(t.std(ddof=1)) if len(t) > 1 else 0.0, 4),
            "rel_std": round(float(t.std(ddof=1) / t.mean()) if len(t) > 1 else 0.0, 5),
            "min_ms": round(float(t.min()), 4), "max_ms": round(float(t.max()), 4), "n": int(len(t))}


def emit_c2(args, res_all, rank, world):
    peaks, peak_src = measured_peaks()
    r0 = res_all[0]
    # max over ranks of the device-timed region; value = all ranks' useful
    # read bytes (4 B per read) / that time
    tmax = max(r["total_t"] for r in res_all)
    reads = r0["reads"]
    value = sum(r["reads"] * 4 * len(r["times"]) for r in res_all) / tmax / 1e9
    st = r0["stats"][-1]
    per_launch_fill = r0["total_fill"] / len(r0["times"])
    avg_t = r0["total_t"] / len(r0["times"])
    achieved = per_launch_fill / avg_t / 1e9
    e2e_t = max(sum(r["e2e_t"]) for r in res_all)
    e2e_val = sum(r["reads"] * 4 * len(r["e2e_t"]) for r in res_all) / e2e_t / 1e9
    hit = r0["hit"]
    line = {
        "metric": METRIC,
        "value": round(value, 6),
        "unit": "GB/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(tmax / args.steps * 1e3, 3),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "u32",
        "data": "synthetic (splitmix64 file words, seeded uniform offsets)",
        "value_note": "useful apointer read bytes (4 B per read) per second of the device-timed "
                      "step, the reference arm's unit; C2 is fault-bound by construction (one "
                      "64 KiB page fill per missing 4-B read over the host link), so the fault "
                      "path's fill rate against the host link is the roofline below",
        "config": {"workload": r0["cfgd"]["workload"], "file_bytes": r0["cfgd"]["file_bytes"],
                   "page_bytes": r0["cfgd"]["page"], "cache_bytes": r0["cfgd"]["frames"] *
                   r0["cfgd"]["page"], "reads_per_step": reads, "elem_bytes": 4,
                   "grid": r0["cfgd"]["grid"], "block": r0["cfgd"]["block"],
                   "l2": "inputs larger than L2 (4 GiB file, 1 GiB cache, 126 MB L2); cache "
                         "reset (cold) before every step",
                   "parallelism": f"replicas x{world} (one cache + file per GPU)"},
        "step_times": step_stats(r0["times"]),
        "fault_bound": {
            "fill_GBps": round(achieved, 3),
            "host_link_GBps_memcpy": round(r0["link"], 2),
            "host_link_GBps_zero_copy_sm": round(r0["zc_gbs"], 2),
            "frac_of_host_link": round(achieved / r0["link"], 4),
            "reads_per_s": round(reads / avg_t, 1),
            "useful_GBps": round(reads * 4 / avg_t / 1e9, 6),
            "fill_bytes_per_useful_byte": round(per_launch_fill / (reads * 4), 1),
            "major_faults": st["major"], "minor_faults": st["minor"],
            "evictions": st["evictions"], "hit_ratio": round(1 - st["major"] / reads, 4),
            "waits": st["waits"], "downgrades": st["downgrades"],
            "raw_zero_copy_twin_s": round(r0["raw_t"], 6),
            "raw_zero_copy_twin_useful_GBps": round(reads * 4 / r0["raw_t"] / 1e9, 6),
            "raw_twin_checksums_equal": r0["raw_match"],
            "device_error": r0["err"]},
        "hit": {
            "workload": "1 GiB resident (prefilled), SEQ 16-B apointer reads, each warp walks "
                        "whole 64 KiB pages (PAPER.md:367), 8 passes, all SMs",
            "apointer_GBps": round(hit["tile"]["gbs"], 1), "raw_GBps": round(hit["raw_gbs"], 1),
            "overhead_vs_raw": round(hit["tile"]["overhead"], 4),
            "frac_of_hbm": round(hit["tile"]["gbs"] / peaks["hbm_gbs"], 4),
            "hbm_peak_GBps": peaks["hbm_gbs"], "peak_source": peak_src,
            "access_styles": {k: {"GBps": round(hit[k]["gbs"], 1),
                                  "overhead_vs_raw": round(hit[k]["overhead"], 4)}
                              for k in ("tile", "range", "deref")},
            "deref_vs_raw_per_access_twin": {
                "raw_GBps": round(hit["deref"]["raw_deref_gbs"], 1),
                "overhead": round(hit["deref"]["overhead_vs_raw_deref"], 4),
                "grid": hit["deref"]["grid"]},
            "access_note": "tile = read_tile<16> (one translation check per 16 accesses, the "
                           "headline); range = pin_range (one check per page); deref = `v = *q; "
                           "q += 32` one access at a time (the paper's loop, each access checked "
                           "and able to fault; the loop issues access j+D before it uses access "
                           "j, D = AP_DEREF_PIPE = 8, 148 CTAs of 512), overhead_vs_raw is "
                           "against the tiled raw "
                           "twin, deref_vs_raw_per_access_twin against the identical per-access "
                           "loop on a raw pointer at the same launch",
            "overhead_method": "median over %d alternating (apointer, raw) launch pairs of "
                               "t_apointer / t_raw - 1 (CUDA events on the launch stream; 1 GiB "
                               "per launch > L2)" % hit["pairs"],
            "major_faults_during": hit["majors_during"],
            "checksums_equal_raw": hit["checksums_equal_raw"]},
        "minor": {
            "workload": "M2r: the same resident GiB, uniform-random 4-B apointer reads (8 per "
                        "thread, 4x148 CTAs of 512): every read leaves its page, i.e. one unlink "
                        "+ one minor fault (PTE atomic) per read; raw twin = the same gather "
                        "from an HBM copy",
            "reads_per_s": round(hit["minor"]["reads_per_s"], 1),
            "raw_reads_per_s": round(hit["minor"]["raw_reads_per_s"], 1),
            "useful_GBps": round(hit["minor"]["useful_gbs"], 3),
            "sector_GBps": round(hit["minor"]["sector_gbs"], 3),
            "overhead_vs_raw": round(hit["minor"]["overhead"], 4),
            "ceiling_reads_per_s": (hit["minor"]["ceiling"] or {}).get(
                "acquire add + 4-B gather + release add"),
            "frac_of_ceiling": (round(hit["minor"]["reads_per_s"] /
                                      hit["minor"]["ceiling"]["acquire add + 4-B gather + release add"], 4)
                                if hit["minor"].get("ceiling") else None),
            "ceiling_note": "tools/atomic_ceiling, run in this session: per read one acquire add "
                            "and one release add on random entries of a 16 384-entry PTE array "
                            "plus the 4-B gather, no page-cache logic (all G steps/s: "
                            "%s)" % {k: round(v / 1e9, 2) for k, v in
                                     (hit["minor"].get("ceiling") or {}).items()},
            "major_faults_during": hit["minor"]["majors"],
            "minor_faults_per_launch": hit["minor"]["minors_per_launch"],
            "checksums_equal_raw": hit["minor"]["equal_raw"]},
        "roofline": {"bound": "host_link", "achieved": round(achieved, 3),
                     "peak": round(r0["link"], 3), "unit": "GB/s",
                     "frac": round(achieved / r0["link"], 4),
                     "traffic": ncu_traffic("k_random<uint32_t, UNIFORM, apointer>"),
                     "algorithmic_bytes_per_launch": int(per_launch_fill),
                     "kernel": "k_random<uint32_t, UNIFORM, apointer>",
                     "achieved_note": "page-fill bytes the fault path moved over the host link "
                                      "per launch / mean CUDA-event launch time",
                     "peak_source": "host->device cudaMemcpy from pinned memory, measured in this "
                                    "run (no host-link entry in MEASURED_PEAKS.json)"},
        "e2e": {"value": round(e2e_val, 6), "unit": "GB/s",
                "h2d_bytes_per_step": int(r0["e2e_fill"] / len(r0["e2e_t"])),
                "d2h_bytes_per_step": r0["nthreads"] * 8,
                "api": "ap_bench_read_host (launch + device->host copy of the checksums); "
                       "useful read bytes per second like value.  h2d = the page bytes the "
                       "fault path pulls from the pinned host file inside the step (zero-copy "
                       "16-B loads over PCIe, not a cudaMemcpy): the file never sits in HBM "
                       "before the step",
                "checksums_equal_device_run": r0["e2e_match"]},
        "gpu_launches": args.steps,
        "clocks": r0["clocks"],
    }
    if world == 1 and not args.no_cpu_baseline:
        threads = os.cpu_count() or 1
        dt, match, npass = cpu_oracle_c2(r0, threads)
        line["cpu_baseline"] = {"value": round(reads * 4 / dt / 1e9, 6), "unit": "GB/s",
                                "cores": threads, "kind": "oracle",
                                "sample": f"{npass} passes of a full C2-sized read set ({reads} "
                                          f"uniform 4-B reads of the 4 GiB file + FNV-1a per "
                                          f"thread, fresh seed per pass), {dt:.4f} s per pass; "
                                          f"value = bytes read / s (the oracle has no pages to "
                                          f"fill); bench seed checksums equal GPU: {match}"}
    return line


# ------------------------------------------------------------------ reference arm
def run_reference(args):
    rank, _, world = env_rank()
    if rank != 0:
        return
    import oracle
    import synth
    cfgd = c2_config(args)
    f = synth.fill_file(aligned_empty(cfgd["file_bytes"]), cfgd["file_seed"])
    nthreads = cfgd["grid"] * cfgd["block"]
    threads = os.cpu_count() or 1
    ts = []
    for i in range(args.warmup + args.steps):
        t0 = time.time()
        oracle.read_uniform(f, cfgd["file_bytes"], 4, nthreads, cfgd["reads_per_thread"],
                            cfgd["seed"], threads=threads)
        if i >= args.warmup:
            ts.append(time.time() - t0)
    reads = nthreads * cfgd["reads_per_thread"]
    dt = float(np.mean(ts))
    v = reads * 4 / dt / 1e9
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(v, 6), "unit": "GB/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(dt * 1e3, 3), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": cfgd["workload"]},
        "cpu_baseline": {"value": round(v, 6), "unit": "GB/s", "cores": threads,
                         "kind": "oracle",
                         "sample": f"each step = the full C2 read set ({reads} reads), plain file "
                                   f"indexing on the host cores; bytes = 4 per read"},
        "e2e": {"value": round(v, 6), "unit": "GB/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0}}), flush=True)


def gather_all(res, drop, rank, world, dist):
    """Every rank's result dict on rank 0 (rank 0 keeps its own in full)."""
    if world == 1:
        return [res]
    gathered = [None] * world
    slim = {k: v for k, v in res.items() if k not in drop}
    dist.all_gather_object(gathered, slim)
    return [res] + gathered[1:] if rank == 0 else gathered


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--workload", default="c2", choices=["c1", "c2", "c3", "c4", "c5"])
    p.add_argument("--group", type=int, default=8, help="collage candidates per warp (1, 2, 4, 8)")
    p.add_argument("--schedule", type=int, default=2, help="collage: 0 = natural, 1 = LSH-sorted blocks, 2 = per-table units, 3 = per-table units in bucket-MinHash order")
    p.add_argument("--stride", type=int, default=4096, help="collage record stride (3072 = unaligned)")
    p.add_argument("--partition", default="records", choices=["records", "units", "blocks"],
                   help="collage, N > 1, per-table schedules: split the record ids (each GPU "
                        "caches one shard of the file), the sorted units, or the image")
    p.add_argument("--id-chunks", type=int, default=None,
                   help="collage record-id windows (ap_collage_in.id_chunks; 0 = off; "
                        "default 32 for c4, 96 for c5 (fused windows; measured C4 12/32/64 -> "
                        "28.1/27.1/27.1 ms, C5 12/24/48/96 -> 0.589/0.541/0.495/0.486 s, "
                        "profiles/r02_collage_warp_units.txt)")
    p.add_argument("--reads", type=int, default=8, help="reads per thread (C2)")
    p.add_argument("--policy", default=None, choices=["clock", "sequential"],
                   help="c1/c3 eviction policy (default: sequential drop-behind for the "
                        "single-pass c1 stream, clock otherwise)")
    p.add_argument("--combine", default="fused", choices=["fused", "nccl"],
                   help="collage, N > 1: fold winners into rank 0's array from the kernels "
                        "(CUDA IPC + system-scope atomics, no collective) or one NCCL "
                        "gather / MIN reduce after the kernel")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-c5", action="store_true",
                   help="default workload only: skip the embedded C5 collage object (40 GB host file)")
    p.add_argument("--no-reads", action="store_true",
                   help="default workload only: skip the embedded C1 / C3 objects")
    p.add_argument("--no-collage", action="store_true",
                   help="default workload only: skip the embedded C4 collage object")
    args = p.parse_args()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    rank, local, world = env_rank()
    # AP_BENCH_SHARE_GPU=1 (validation only): every rank on cuda:0 with gloo
    # collectives, to exercise the N>1 code paths on a one-GPU box.  Timings
    # from such a run are not bench numbers.
    share = os.environ.get("AP_BENCH_SHARE_GPU") == "1"
    local_dev = 0 if share else local
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    if os.environ.get("AP_NUMA_LOCAL", "1") == "1":
        node = gpu_numa_node(torch, dev)
        if node is not None:
            os.environ["AP_BENCH_NODE"] = str(node)
    dist = None
    if world > 1:
        import torch.distributed as dist
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    if args.workload in ("c4", "c5"):
        import bench_collage
        res = bench_collage.run_collage(args, torch, dev, rank, world, dist, timed, ClockSampler,
                                        host_link_peak)
        drop = ("got", "is_copy", "src")
    elif args.workload in ("c1", "c3"):
        import bench_reads
        res = bench_reads.run_reads(args, torch, dev, rank, world, dist, timed, ClockSampler,
                                    host_link_peak, aligned_empty)
        drop = ()
    else:
        res = run_c2(args, torch, dev, rank, world, dist)
        drop = ("file", "got")
    coll_all = None
    if args.workload == "c2" and not args.no_collage:
        # the C4 collage rides along in the default line (BASELINE.json
        # configs[3]; the metric's "collage s"): one cold step per timed step
        import copy
        import bench_collage
        cargs = copy.copy(args)
        cargs.workload, cargs.stride = "c4", 4096
        cres = bench_collage.run_collage(cargs, torch, dev, rank, world, dist, timed, ClockSampler,
                                         host_link_peak, light=True)
        coll_all = gather_all(cres, ("got", "is_copy", "src"), rank, world, dist)
        del cres
    c5_all = None
    if args.workload == "c2" and not args.no_collage and not args.no_c5:
        # and C5 (configs[4]: 10M records, 40 GB pinned file, the multi-GPU
        # collage; one step per timed step at this --gpus N)
        import copy
        import bench_collage
        c5args = copy.copy(args)
        c5args.workload, c5args.stride = "c5", 4096
        c5res = bench_collage.run_collage(c5args, torch, dev, rank, world, dist, timed, ClockSampler,
                                          host_link_peak, light=True)
        c5_all = gather_all(c5res, ("got", "is_copy", "src"), rank, world, dist)
        del c5res
    reads_all = {}
    if args.workload == "c2" and not args.no_reads:
        # C1 and C3 (BASELINE.json configs[0], [2]: the paper's page-fault
        # microbenchmark regimes) ride along as well
        import copy
        import bench_reads
        for w in ("c1", "c3"):
            rargs = copy.copy(args)
            rargs.workload, rargs.policy = w, None
            rres = bench_reads.run_reads(rargs, torch, dev, rank, world, dist, timed, ClockSampler,
                                         host_link_peak, aligned_empty)
            reads_all[w] = (rargs, gather_all(rres, (), rank, world, dist))
    res_all = gather_all(res, drop, rank, world, dist)
    if rank == 0:
        if args.workload in ("c4", "c5"):
            line = bench_collage.emit_collage(args, res_all, world, METRIC)
        elif args.workload in ("c1", "c3"):
            line = bench_reads.emit_reads(args, res_all, world, METRIC)
        else:
            line = emit_c2(args, res_all, rank, world)
            if coll_all is not None:
                import copy
                import bench_collage
                cargs = copy.copy(args)
                cargs.workload = "c4"
                line["collage_c4"] = bench_collage.collage_summary(cargs, coll_all, world)
            if c5_all is not None:
                import copy
                import bench_collage
                c5args = copy.copy(args)
                c5args.workload = "c5"
                line["collage_c5"] = bench_collage.collage_summary(c5args, c5_all, world)
            for w, (rargs, rall) in reads_all.items():
                import bench_reads
                line[f"reads_{w}"] = bench_reads.reads_summary(rargs, rall, world, METRIC)
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
