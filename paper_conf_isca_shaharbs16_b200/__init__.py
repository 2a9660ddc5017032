"""ActivePointers on B200 -- Python binding of libapointer.so (include/ap.h).

Same names as the C ABI; arguments are marshalled, nothing is computed here.
Device buffers are torch CUDA tensors (PyTorch provides memory and streams
only); host buffers are numpy arrays or torch CPU tensors.
"""
import ctypes

import numpy as np

from . import _lib
from ._lib import (AP_PROT_READ, AP_PROT_WRITE, AP_ACCESS_DEREF, AP_ACCESS_RANGE, AP_ACCESS_AHEAD, AP_ACCESS_PAIR, AP_ACCESS_TMA, AP_ACCESS_TILE, AP_DIVERGENT, AP_MODE_APOINTER, AP_MODE_RAW, AP_POLICY_CLOCK, AP_POLICY_SEQUENTIAL,  # noqa: F401
                   AP_POLICY_RANDOM, AP_SCHED_LSH, AP_SCHED_NATURAL, AP_SCHED_TABLE, AP_SCHED_TABLE_MH, AP_SEQ, AP_SEQ_QUEUE,
                   AP_UNIFORM, APError, ap_bench_cfg, ap_collage_in,
                   ap_stats_t, AP_COLLAGE_ACCUMULATE, AP_COLLAGE_SYSTEM, AP_PART_BLOCKS,
                   AP_PART_RECORDS, AP_PART_UNITS, AP_MGPU_MAX, ap_ipc_handle_t,
                   ap_mgpu_collage_in, ap_mgpu_report)

_frames = {}


def _ptr(buf):
    """Address of a numpy array / torch tensor / raw int."""
    if buf is None:
        return None
    if isinstance(buf, int):
        return buf
    if isinstance(buf, np.ndarray):
        return buf.ctypes.data
    if hasattr(buf, "data_ptr"):
        return buf.data_ptr()
    raise TypeError(f"cannot take the address of {type(buf)}")


def _nbytes(buf):
    if isinstance(buf, np.ndarray):
        return buf.nbytes
    if hasattr(buf, "element_size"):
        return buf.numel() * buf.element_size()
    raise TypeError(type(buf))


def _stream(stream):
    if stream is None:
        try:
            import torch
            if torch.cuda.is_available():
                return torch.cuda.current_stream().cuda_stream
        except Exception:
            pass
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def ap_version():
    return _lib.lib().ap_version().decode()


def ap_strerror(code):
    return _lib.lib().ap_strerror(code).decode()


def ap_cache_create(frames, page_size, device=0):
    h = ctypes.c_void_p()
    _lib.check("ap_cache_create", _lib.lib().ap_cache_create(frames, page_size, device,
                                                             ctypes.byref(h)))
    _frames[h.value] = frames
    return h.value


def ap_cache_destroy(cache):
    _lib.check("ap_cache_destroy", _lib.lib().ap_cache_destroy(cache))
    _frames.pop(cache, None)


def ap_mmap(cache, host_buf, nbytes=None):
    r = ctypes.c_uint32()
    nbytes = _nbytes(host_buf) if nbytes is None else nbytes
    _lib.check("ap_mmap", _lib.lib().ap_mmap(cache, _ptr(host_buf), nbytes, ctypes.byref(r)))
    return r.value


def ap_mmap_prot(cache, host_buf, prot, nbytes=None):
    r = ctypes.c_uint32()
    nbytes = _nbytes(host_buf) if nbytes is None else nbytes
    _lib.check("ap_mmap_prot", _lib.lib().ap_mmap_prot(cache, _ptr(host_buf), nbytes, prot,
                                                       ctypes.byref(r)))
    return r.value


def ap_msync(cache, region):
    _lib.check("ap_msync", _lib.lib().ap_msync(cache, region))


def ap_munmap(cache, region):
    _lib.check("ap_munmap", _lib.lib().ap_munmap(cache, region))


def ap_region_devptr(cache, region):
    p = ctypes.c_void_p()
    _lib.check("ap_region_devptr", _lib.lib().ap_region_devptr(cache, region, ctypes.byref(p)))
    return p.value


def ap_region_add_peer(cache, region, peer, peer_region):
    """N2: major faults of `region` copy pages resident in `peer_region` of
    the cache `peer` (same process; same or peer-accessible GPU)."""
    _lib.check("ap_region_add_peer", _lib.lib().ap_region_add_peer(cache, region, peer, peer_region))


def ap_region_export(cache, region):
    """N2 across processes: the region's peer record as bytes (CUDA IPC
    handles + sizes), to hand to ap_region_add_peer_ipc in another process."""
    h = _lib.ap_peer_handle_t()
    _lib.check("ap_region_export", _lib.lib().ap_region_export(cache, region, ctypes.byref(h)))
    return bytes(h)


def ap_region_add_peer_ipc(cache, region, handle):
    h = _lib.ap_peer_handle_t.from_buffer_copy(bytes(handle))
    _lib.check("ap_region_add_peer_ipc",
               _lib.lib().ap_region_add_peer_ipc(cache, region, ctypes.byref(h)))


def ap_region_clear_peers(cache, region):
    _lib.check("ap_region_clear_peers", _lib.lib().ap_region_clear_peers(cache, region))


def ap_region_npages(cache, region):
    n = ctypes.c_uint64()
    _lib.check("ap_region_npages", _lib.lib().ap_region_npages(cache, region, ctypes.byref(n)))
    return n.value


def ap_cache_stats(cache):
    s = ap_stats_t()
    _lib.check("ap_cache_stats", _lib.lib().ap_cache_stats(cache, ctypes.byref(s)))
    return s.as_dict()


def ap_cache_reset(cache):
    _lib.check("ap_cache_reset", _lib.lib().ap_cache_reset(cache))


def ap_cache_set_policy(cache, policy, seed=0):
    _lib.check("ap_cache_set_policy", _lib.lib().ap_cache_set_policy(cache, policy, seed))


def ap_cache_set_tuning(cache, max_claims=1, sweep_steps=64, timeout_ms=0):
    _lib.check("ap_cache_set_tuning",
               _lib.lib().ap_cache_set_tuning(cache, max_claims, sweep_steps, timeout_ms))


def ap_cache_set_backoff(cache, min_ns=64, max_ns=4096):
    _lib.check("ap_cache_set_backoff", _lib.lib().ap_cache_set_backoff(cache, min_ns, max_ns))


def ap_last_device_error(cache):
    return _lib.lib().ap_last_device_error(cache)


def ap_cache_dump(cache):
    frames = _frames[cache]
    owner = np.empty(frames, dtype=np.uint64)
    left = ctypes.c_uint64()
    _lib.check("ap_cache_dump", _lib.lib().ap_cache_dump(cache, owner.ctypes.data,
                                                         ctypes.byref(left)))
    return owner, left.value


def ap_region_dump_pte(cache, region):
    pte = np.empty(ap_region_npages(cache, region), dtype=np.uint64)
    _lib.check("ap_region_dump_pte", _lib.lib().ap_region_dump_pte(cache, region,
                                                                   pte.ctypes.data))
    return pte


def ap_prefill(cache, region, first_page, npages, stream=None):
    _lib.check("ap_prefill", _lib.lib().ap_prefill(cache, region, first_page, npages,
                                                   _stream(stream)))


def bench_cfg(pattern, elem_bytes, grid, block, reads_per_thread=0, passes=1, unit_bytes=0,
              page_bytes=0, span_bytes=0, seed=0, mode=AP_MODE_APOINTER, out_copy=False,
              raw_base=None, access=AP_ACCESS_TILE):
    return ap_bench_cfg(pattern, elem_bytes, grid, block, reads_per_thread, passes, unit_bytes,
                        page_bytes, span_bytes, seed, mode, int(out_copy), raw_base, access)


def ap_bench_read(cache, region, cfg, out_dev, stream=None):
    _lib.check("ap_bench_read", _lib.lib().ap_bench_read(cache, region, ctypes.byref(cfg),
                                                         _ptr(out_dev), _stream(stream)))


def ap_bench_write(cache, region, cfg, stream=None):
    _lib.check("ap_bench_write", _lib.lib().ap_bench_write(cache, region, ctypes.byref(cfg),
                                                           _stream(stream)))


def ap_bench_copy(cache, src, dst, cfg, stream=None):
    _lib.check("ap_bench_copy", _lib.lib().ap_bench_copy(cache, src, dst, ctypes.byref(cfg),
                                                         _stream(stream)))


def ap_bench_read_host(cache, region, cfg, out_host):
    sec = ctypes.c_double()
    _lib.check("ap_bench_read_host", _lib.lib().ap_bench_read_host(
        cache, region, ctypes.byref(cfg), _ptr(out_host), ctypes.byref(sec)))
    return sec.value


WORKS = {"add": 0, "read": 1, "random": 2, "reduce": 3, "fft": 4, "bitonic": 5}


def ap_bench_compute(cache, region, work, elem_bytes, grid, block, span_bytes, out_dev, iters=0,
                     mode=AP_MODE_APOINTER, raw_base=None, stream=None):
    cfg = _lib.ap_compute_cfg(WORKS.get(work, work), elem_bytes, grid, block, iters, span_bytes,
                              mode, _ptr(raw_base))
    _lib.check("ap_bench_compute", _lib.lib().ap_bench_compute(cache, region, ctypes.byref(cfg),
                                                               _ptr(out_dev), _stream(stream)))


def ap_bench_latency(cache, region, op, reps=1000):
    """Returns (cycles per op, empty timing-pair cycles)."""
    out = (ctypes.c_uint64 * 2)()
    _lib.check("ap_bench_latency", _lib.lib().ap_bench_latency(cache, region, op, reps, out))
    return int(out[0]), int(out[1])


def collage_in(target_dev, W, H, proj_dev, bias_dev, w, bucket_bits, offsets_dev, ids_dev, N,
               rec_stride=4096, group=1, block_begin=0, block_count=None,
               mode=AP_MODE_APOINTER, raw_base=None, L=None, K=None, schedule=AP_SCHED_TABLE,
               unit_begin=0, unit_count=0, id_chunks=0, id_begin=0, id_end=0, flags=0):
    L = proj_dev.shape[0] if L is None else L
    K = proj_dev.shape[1] if K is None else K
    nb = (W // 32) * (H // 32)
    block_count = nb - block_begin if block_count is None else block_count
    return ap_collage_in(_ptr(target_dev), W, H, L, K, bucket_bits, w, _ptr(proj_dev),
                         _ptr(bias_dev), _ptr(offsets_dev), _ptr(ids_dev), N, rec_stride, group,
                         block_begin, block_count, mode, _ptr(raw_base), schedule, unit_begin,
                         unit_count, id_chunks, id_begin, id_end, flags)


def ap_collage_run(cache, region, inp, winners_dev, stream=None):
    _lib.check("ap_collage_run", _lib.lib().ap_collage_run(cache, region, ctypes.byref(inp),
                                                           _ptr(winners_dev), _stream(stream)))


def ap_winners_init(winners_dev, nblocks, stream=None):
    _lib.check("ap_winners_init", _lib.lib().ap_winners_init(_ptr(winners_dev), nblocks,
                                                             _stream(stream)))


def ap_ipc_export(dev_buf):
    """CUDA IPC handle (ap_ipc_handle_t) of a device buffer of this process."""
    h = ap_ipc_handle_t()
    _lib.check("ap_ipc_export", _lib.lib().ap_ipc_export(_ptr(dev_buf), ctypes.byref(h)))
    return h


def ap_ipc_import(handle, device):
    """Map another process's buffer on `device`; returns its device address."""
    out = ctypes.c_void_p()
    _lib.check("ap_ipc_import", _lib.lib().ap_ipc_import(ctypes.byref(handle), device,
                                                         ctypes.byref(out)))
    return out.value


def ap_ipc_close(dev_ptr):
    _lib.check("ap_ipc_close", _lib.lib().ap_ipc_close(dev_ptr))


def mgpu_collage_in(target_host, W, H, proj_host, bias_host, w, bucket_bits, N, rec_stride=4096,
                    group=8, schedule=AP_SCHED_TABLE, id_chunks=0, partition=AP_PART_RECORDS):
    """Host-side inputs of the multi-GPU collage (the arrays must stay alive
    while the struct is used)."""
    L, K = bias_host.shape
    return ap_mgpu_collage_in(_ptr(target_host), W, H, L, K, bucket_bits, w, _ptr(proj_host),
                              _ptr(bias_host), N, rec_stride, group, schedule, id_chunks,
                              partition)


def ap_mgpu_create(devices, host_file, frames_per_gpu, page_size):
    devs = (ctypes.c_int * len(devices))(*devices)
    out = ctypes.c_void_p()
    _lib.check("ap_mgpu_create", _lib.lib().ap_mgpu_create(
        len(devices), devs, _ptr(host_file), _nbytes(host_file), frames_per_gpu, page_size,
        ctypes.byref(out)))
    return out.value


def ap_mgpu_collage(m, inp, winners_host):
    """One cold step; winners_host = uint32[blocks, 2] host array.  Returns
    the report as a dict."""
    rep = ap_mgpu_report()
    _lib.check("ap_mgpu_collage", _lib.lib().ap_mgpu_collage(m, ctypes.byref(inp),
                                                             _ptr(winners_host),
                                                             ctypes.byref(rep)))
    return rep.as_dict()


def ap_mgpu_destroy(m):
    _lib.check("ap_mgpu_destroy", _lib.lib().ap_mgpu_destroy(m))


def ap_collage_mgpu(devices, host_file, frames_per_gpu, page_size, inp, winners_host):
    devs = (ctypes.c_int * len(devices))(*devices)
    rep = ap_mgpu_report()
    _lib.check("ap_collage_mgpu", _lib.lib().ap_collage_mgpu(
        len(devices), devs, _ptr(host_file), _nbytes(host_file), frames_per_gpu, page_size,
        ctypes.byref(inp), _ptr(winners_host), ctypes.byref(rep)))
    return rep.as_dict()


def ap_lsh_build_index(cache, region, N, rec_stride, L, K, bucket_bits, w, proj_dev, bias_dev,
                       offsets_dev, ids_dev, stream=None):
    _lib.check("ap_lsh_build_index", _lib.lib().ap_lsh_build_index(
        cache, region, N, rec_stride, L, K, bucket_bits, w, _ptr(proj_dev), _ptr(bias_dev),
        _ptr(offsets_dev), _ptr(ids_dev), _stream(stream)))
