"""Fault-path phase breakdown for C1-like SEQ copies (diagnostic build
AP_FAULT_PROF: AP_LIB_PATH=build/variants/lib_fprof.so).  Prints SM cycles per
deref_slow call and per phase, summed over warps, for several frame/grid
points."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_isca_shaharbs16_b200 as ap
from paper_conf_isca_shaharbs16_b200 import _lib
import synth

NAMES = ["calls", "A probe+claim", "B alloc", "C fill", "C fence+publish", "D link/value",
         "deref_slow total", "rounds", "drop_stale", "link_minor", "relinks"]


def aligned_empty(n, align=4096):
    raw = np.empty(n + align, dtype=np.uint8)
    off = (-raw.ctypes.data) % align
    return raw[off:off + n]


def prof(L, reset):
    buf = (ctypes.c_uint64 * 16)()
    rc = L.ap_fault_prof(buf, reset)
    assert rc == 0, rc
    return list(buf)


def main():
    L = _lib.lib()
    L.ap_fault_prof.argtypes = [ctypes.POINTER(ctypes.c_uint64), ctypes.c_int]
    L.ap_fault_prof.restype = ctypes.c_int
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream()
    fb = 16 << 20
    f = synth.fill_file(aligned_empty(fb), 1)
    pts = [tuple(int(v) for v in p.split("x")) for p in
           os.environ.get("AP_EXP_POINTS", "4096x64,64x64,64x148,65x148,148x148,4096x148").split(",")]
    for frames, grid in pts:
        cache = ap.ap_cache_create(frames, 4096, 0)
        region = ap.ap_mmap(cache, f)
        ap.ap_cache_set_policy(cache, ap.AP_POLICY_SEQUENTIAL)
        out = torch.empty(fb, dtype=torch.uint8, device=dev)
        bc = ap.bench_cfg(int(os.environ.get("AP_EXP_PATTERN", ap.AP_SEQ)), 16, grid, 32, unit_bytes=4096, out_copy=True)
        for it in range(3):
            ap.ap_cache_reset(cache)
            torch.cuda.synchronize()
            prof(L, 1)
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            ap.ap_bench_read(cache, region, bc, out, stream)
            e1.record(stream)
            e1.synchronize()
        t = e0.elapsed_time(e1) / 1e3
        p = prof(L, 1)
        st = ap.ap_cache_stats(cache)
        ok = bool(np.array_equal(out.cpu().numpy(), f))
        calls = max(p[0], 1)
        print(f"frames={frames} grid={grid} t={t*1e3:.3f} ms fills={st['fill_bytes']/t/1e9:.2f} GB/s "
              f"major={st['major']} waits={st['waits']} ok={ok}")
        print("   per deref_slow call (cycles): " + ", ".join(
            f"{NAMES[i]}={p[i]/calls:.0f}" for i in (1, 2, 3, 4, 5, 6)) + f", rounds/call={p[7]/calls:.2f}")
        rl = max(p[10], 1)
        print(f"   per relink: drop_stale={p[8]/rl:.0f} link_minor={p[9]/rl:.0f} relinks={p[10]} calls={p[0]}")
        ap.ap_munmap(cache, region)
        ap.ap_cache_destroy(cache)


if __name__ == "__main__":
    main()
