"""C1 characterisation: fills GB/s of the SEQ copy vs frames and grid
(4 KiB pages, 16 MiB file, one warp per block, drop-behind policy)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_isca_shaharbs16_b200 as ap
import synth


def aligned_empty(n, align=4096):
    raw = np.empty(n + align, dtype=np.uint8)
    off = (-raw.ctypes.data) % align
    return raw[off:off + n]


def main():
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream()
    fb = int(os.environ.get("AP_EXP_FILE_MB", 16)) << 20
    f = synth.fill_file(aligned_empty(fb), 1)
    pol = int(os.environ.get("AP_EXP_POLICY", ap.AP_POLICY_SEQUENTIAL))
    fl = [int(v) for v in os.environ.get("AP_EXP_FRAMES", "64,96,128,148,192,256,512,4096").split(",")]
    gl = [int(v) for v in os.environ.get("AP_EXP_GRIDS", "64,148,296").split(",")]
    for frames in fl:
        for grid in gl:
            cache = ap.ap_cache_create(frames, 4096, 0)
            region = ap.ap_mmap(cache, f)
            ap.ap_cache_set_policy(cache, pol)
            if os.environ.get("AP_EXP_BACKOFF"):
                lo, hi = (int(v) for v in os.environ["AP_EXP_BACKOFF"].split(","))
                ap.ap_cache_set_backoff(cache, lo, hi)
            if os.environ.get("AP_EXP_SWEEP"):
                ap.ap_cache_set_tuning(cache, 1, int(os.environ["AP_EXP_SWEEP"]), 0)
            out = torch.empty(fb, dtype=torch.uint8, device=dev)
            bc = ap.bench_cfg(int(os.environ.get("AP_EXP_PATTERN", ap.AP_SEQ)), 16, grid, 32, unit_bytes=4096, out_copy=True)
            ts = []
            for it in range(6):
                ap.ap_cache_reset(cache)
                torch.cuda.synchronize()
                e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                ap.ap_bench_read(cache, region, bc, out, stream)
                e1.record(stream)
                e1.synchronize()
                if it >= 2:
                    ts.append(e0.elapsed_time(e1) / 1e3)
            st = ap.ap_cache_stats(cache)
            ok = bool(np.array_equal(out.cpu().numpy(), f))
            t = min(ts)
            print(f"frames={frames:5d} grid={grid:4d} t={t*1e3:.3f} ms fills={st['fill_bytes']/t/1e9:6.2f} GB/s "
                  f"waits={st['waits']} nofree={st['nofree']} evict={st['evictions']} ok={ok}", flush=True)
            ap.ap_munmap(cache, region)
            ap.ap_cache_destroy(cache)


if __name__ == "__main__":
    main()
