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
