"""ctypes binding of libapointer.so (include/ap.h). Argument marshalling only:
every step of the path runs in the library's CUDA kernels.

Fails loudly when the library is missing -- there is no CPU fallback.
"""
import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("AP_LIB_PATH") or os.path.join(_HERE, "libapointer.so")

AP_OK = 0
AP_EINVAL, AP_ENOMEM, AP_ECUDA, AP_EBUSY, AP_ERANGE = -1, -2, -3, -4, -5
AP_EFAULT, AP_ENOFRAME, AP_ETIMEDOUT = -6, -7, -8
AP_POLICY_CLOCK, AP_POLICY_RANDOM, AP_POLICY_SEQUENTIAL = 0, 1, 2
AP_SEQ, AP_UNIFORM, AP_DIVERGENT, AP_SEQ_QUEUE = 0, 1, 2, 3
AP_MODE_APOINTER, AP_MODE_RAW = 0, 1
AP_ACCESS_TILE, AP_ACCESS_DEREF, AP_ACCESS_RANGE, AP_ACCESS_AHEAD, AP_ACCESS_PAIR, AP_ACCESS_TMA = 0, 1, 2, 3, 4, 5
AP_SCHED_NATURAL, AP_SCHED_LSH, AP_SCHED_TABLE, AP_SCHED_TABLE_MH = 0, 1, 2, 3
AP_PROT_READ, AP_PROT_WRITE = 1, 2
AP_EPERM = -9

u64, u32, i32, vp, ci = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int32, ctypes.c_void_p, ctypes.c_int


class ap_stats_t(ctypes.Structure):
    _fields_ = [(n, u64) for n in ("major", "minor", "fill_bytes", "evictions", "waits",
                                   "downgrades", "nofree", "unlinks", "peer_fills",
                                   "peer_bytes", "backoff_spins", "live_refcnt_sum")] + \
               [("err", ctypes.c_int64)]

    def as_dict(self):
        return {n: int(getattr(self, n)) for n, _ in self._fields_}


class ap_peer_handle_t(ctypes.Structure):
    _fields_ = [("pte_handle", ctypes.c_uint8 * 64), ("pool_handle", ctypes.c_uint8 * 64),
                ("pool_offset", u64), ("bytes", u64), ("page_size", u32), ("device", i32)]


class ap_bench_cfg(ctypes.Structure):
    _fields_ = [("pattern", i32), ("elem_bytes", u32), ("grid", u32), ("block", u32),
                ("reads_per_thread", u32), ("passes", u32), ("unit_bytes", u32),
                ("page_bytes", u32), ("span_bytes", u64), ("seed", u64), ("mode", i32),
                ("out_copy", i32), ("raw_base", vp), ("access", i32)]


class ap_collage_in(ctypes.Structure):
    _fields_ = [("target_dev", vp), ("W", u32), ("H", u32), ("L", u32), ("K", u32),
                ("bucket_bits", u32), ("w", i32), ("proj_dev", vp), ("bias_dev", vp),
                ("offsets_dev", vp), ("ids_dev", vp), ("N", u64), ("rec_stride", u32),
                ("group", u32), ("block_begin", u64), ("block_count", u64), ("mode", i32),
                ("raw_base", vp), ("schedule", i32), ("unit_begin", u64), ("unit_count", u64),
                ("id_chunks", u32), ("id_begin", u32), ("id_end", u32), ("flags", u32)]


AP_COLLAGE_ACCUMULATE, AP_COLLAGE_SYSTEM = 1, 2
AP_PART_BLOCKS, AP_PART_RECORDS, AP_PART_UNITS = 0, 1, 2
AP_MGPU_MAX = 16


class ap_ipc_handle_t(ctypes.Structure):
    _fields_ = [("handle", ctypes.c_uint8 * 64), ("offset", u64), ("bytes", u64),
                ("device", i32), ("pid", i32)]


class ap_mgpu_collage_in(ctypes.Structure):
    _fields_ = [("target_host", vp), ("W", u32), ("H", u32), ("L", u32), ("K", u32),
                ("bucket_bits", u32), ("w", i32), ("proj_host", vp), ("bias_host", vp),
                ("N", u64), ("rec_stride", u32), ("group", u32), ("schedule", i32),
                ("id_chunks", u32), ("partition", i32)]


class ap_mgpu_report(ctypes.Structure):
    _fields_ = [("seconds", ctypes.c_double), ("part_seconds", ctypes.c_double * AP_MGPU_MAX),
                ("fill_bytes", u64 * AP_MGPU_MAX), ("major", u64 * AP_MGPU_MAX),
                ("device_error", i32), ("nparts", i32)]

    def as_dict(self):
        n = self.nparts
        return {"seconds": self.seconds, "part_seconds": list(self.part_seconds[:n]),
                "fill_bytes": [int(x) for x in self.fill_bytes[:n]],
                "major": [int(x) for x in self.major[:n]], "device_error": self.device_error}


class ap_compute_cfg(ctypes.Structure):
    _fields_ = [("work", i32), ("elem_bytes", u32), ("grid", u32), ("block", u32),
                ("iters", u32), ("span_bytes", u64), ("mode", i32), ("raw_base", vp)]


class APError(RuntimeError):
    def __init__(self, fn, code, msg):
        super().__init__(f"{fn} failed: {code} ({msg})")
        self.code = code


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(
                f"{LIB_PATH} is missing: the CUDA extension must be built (`make` or "
                f"__graft_entry__.build()); there is no fallback path")
        L = ctypes.CDLL(LIB_PATH)
        sig = {
            "ap_strerror": (ctypes.c_char_p, [ci]),
            "ap_version": (ctypes.c_char_p, []),
            "ap_cache_create": (ci, [u64, u32, ci, ctypes.POINTER(vp)]),
            "ap_cache_destroy": (ci, [vp]),
            "ap_mmap": (ci, [vp, vp, u64, ctypes.POINTER(u32)]),
            "ap_munmap": (ci, [vp, u32]),
            "ap_region_devptr": (ci, [vp, u32, ctypes.POINTER(vp)]),
            "ap_region_npages": (ci, [vp, u32, ctypes.POINTER(u64)]),
            "ap_cache_stats": (ci, [vp, ctypes.POINTER(ap_stats_t)]),
            "ap_cache_reset": (ci, [vp]),
            "ap_cache_set_policy": (ci, [vp, ci, u64]),
            "ap_cache_set_tuning": (ci, [vp, u32, u32, u32]),
            "ap_cache_set_backoff": (ci, [vp, u32, u32]),
            "ap_last_device_error": (ci, [vp]),
            "ap_cache_dump": (ci, [vp, vp, ctypes.POINTER(u64)]),
            "ap_region_dump_pte": (ci, [vp, u32, vp]),
            "ap_prefill": (ci, [vp, u32, u64, u64, vp]),
            "ap_bench_read": (ci, [vp, u32, ctypes.POINTER(ap_bench_cfg), vp, vp]),
            "ap_bench_read_host": (ci, [vp, u32, ctypes.POINTER(ap_bench_cfg), vp,
                                        ctypes.POINTER(ctypes.c_double)]),
            "ap_collage_run": (ci, [vp, u32, ctypes.POINTER(ap_collage_in), vp, vp]),
            "ap_bench_latency": (ci, [vp, u32, ci, u32, ctypes.POINTER(u64)]),
            "ap_mmap_prot": (ci, [vp, vp, u64, ci, ctypes.POINTER(u32)]),
            "ap_bench_compute": (ci, [vp, u32, ctypes.POINTER(ap_compute_cfg), vp, vp]),
            "ap_msync": (ci, [vp, u32]),
            "ap_bench_write": (ci, [vp, u32, ctypes.POINTER(ap_bench_cfg), vp]),
            "ap_bench_copy": (ci, [vp, u32, u32, ctypes.POINTER(ap_bench_cfg), vp]),
            "ap_region_add_peer": (ci, [vp, u32, vp, u32]),
            "ap_region_export": (ci, [vp, u32, ctypes.POINTER(ap_peer_handle_t)]),
            "ap_region_add_peer_ipc": (ci, [vp, u32, ctypes.POINTER(ap_peer_handle_t)]),
            "ap_region_clear_peers": (ci, [vp, u32]),
            "ap_lsh_build_index": (ci, [vp, u32, u64, u32, u32, u32, u32, i32, vp, vp, vp, vp,
                                        vp]),
            "ap_winners_init": (ci, [vp, u64, vp]),
            "ap_ipc_export": (ci, [vp, ctypes.POINTER(ap_ipc_handle_t)]),
            "ap_ipc_import": (ci, [ctypes.POINTER(ap_ipc_handle_t), ci, ctypes.POINTER(vp)]),
            "ap_ipc_close": (ci, [vp]),
            "ap_mgpu_create": (ci, [ci, ctypes.POINTER(ci), vp, u64, u64, u32,
                                    ctypes.POINTER(vp)]),
            "ap_mgpu_collage": (ci, [vp, ctypes.POINTER(ap_mgpu_collage_in), vp,
                                     ctypes.POINTER(ap_mgpu_report)]),
            "ap_mgpu_destroy": (ci, [vp]),
            "ap_collage_mgpu": (ci, [ci, ctypes.POINTER(ci), vp, u64, u64, u32,
                                     ctypes.POINTER(ap_mgpu_collage_in), vp,
                                     ctypes.POINTER(ap_mgpu_report)]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


EXPORTED = ["ap_strerror", "ap_version", "ap_cache_create", "ap_cache_destroy", "ap_mmap",
            "ap_munmap", "ap_region_devptr", "ap_region_npages", "ap_cache_stats",
            "ap_cache_reset", "ap_cache_set_policy", "ap_cache_set_tuning",
            "ap_last_device_error", "ap_cache_dump", "ap_region_dump_pte", "ap_prefill",
            "ap_bench_read", "ap_bench_read_host", "ap_collage_run", "ap_lsh_build_index",
            "ap_bench_latency", "ap_mmap_prot", "ap_msync", "ap_bench_write", "ap_bench_copy",
            "ap_bench_compute", "ap_cache_set_backoff", "ap_region_add_peer", "ap_region_export",
            "ap_region_add_peer_ipc", "ap_region_clear_peers", "ap_winners_init",
            "ap_ipc_export", "ap_ipc_import", "ap_ipc_close", "ap_mgpu_create",
            "ap_mgpu_collage", "ap_mgpu_destroy", "ap_collage_mgpu"]


def check(fn, rc):
    if rc != AP_OK:
        raise APError(fn, rc, lib().ap_strerror(rc).decode())
    return rc
