"""Shared helpers for the tests (input plumbing only -- no method arithmetic)."""
import numpy as np

import synth


def aligned_empty(nbytes, align=4096):
    raw = np.empty(nbytes + align, dtype=np.uint8)
    off = (-raw.ctypes.data) % align
    return raw[off:off + nbytes]


def make_file(nbytes, seed):
    return synth.fill_file(aligned_empty(nbytes), seed)


def make_records(n, stride, seed):
    return synth.fill_records(aligned_empty(n * stride), 0, n, stride, seed)


def check_invariants(ap, cache, regions, frames, zero_refs=True):
    from oracle import invariants
    owner, free_left = ap.ap_cache_dump(cache)
    ptes = {r: ap.ap_region_dump_pte(cache, r) for r in regions}
    return invariants.check(ptes, owner, free_left, frames, require_zero_refcounts=zero_refs)


def teardown(ap, cache):
    """Unmap whatever regions a (possibly failed) test left mapped, then
    destroy the cache: a region left mapped would keep its host buffer
    registered after Python frees it, and a later buffer at the same address
    would be read through the stale registration."""
    from paper_conf_isca_shaharbs16_b200._lib import APError
    for r in range(64):
        try:
            ap.ap_region_clear_peers(cache, r)
        except APError:
            pass
    for r in range(64):
        try:
            ap.ap_munmap(cache, r)
        except APError:
            pass
    ap.ap_cache_destroy(cache)
