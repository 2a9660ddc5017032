"""Writable mappings (NEXT N3; Fig. 3 `*ptr = 25`): stores
through apointers, DIRTY pages written back on eviction (during the kernel,
with tiny caches), by ap_msync and by ap_munmap.  The host file afterwards
must equal the oracle's plain-indexing application of the same stores."""
import numpy as np
import pytest
import torch

import oracle
from helpers import check_invariants, make_file, teardown

pytestmark = pytest.mark.gpu


def _dirty_count(ap, cache, r):
    pte = ap.ap_region_dump_pte(cache, r)
    return int(((pte >> np.uint64(60)) & np.uint64(1)).sum())


@pytest.mark.parametrize("elem", [4, 16])
@pytest.mark.parametrize("frames", [2, 16, 1024])
def test_seq_writes_reach_the_file(ap, elem, frames):
    n = (1 << 20) + 4096 + 32
    f = make_file(n, seed=1)
    want = oracle.apply_writes(f, elem, 0, span=n, seed=7)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        r = ap.ap_mmap_prot(cache, f, ap.AP_PROT_READ | ap.AP_PROT_WRITE)
        ap.ap_bench_write(cache, r, ap.bench_cfg(ap.AP_SEQ, elem, 4, 128, unit_bytes=4096,
                                                 span_bytes=n, seed=7))
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        st = ap.ap_cache_stats(cache)
        if frames < (n >> 12):
            assert st["evictions"] > 0  # dirty pages went back during the kernel
        ap.ap_msync(cache, r)
        assert _dirty_count(ap, cache, r) == 0
        assert np.array_equal(f, want)
        assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("policy,frames", [(0, 3), (1, 3), (0, 64), (1, 512)])
def test_scattered_writes_then_reads(ap, policy, frames):
    n = 2 << 20
    f = make_file(n, seed=2)
    orig = f.copy()
    want = oracle.apply_writes(orig, 4, 1, nthreads=8 * 256, reads=8, seed=3)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        ap.ap_cache_set_policy(cache, policy, 11)
        r = ap.ap_mmap_prot(cache, f, ap.AP_PROT_READ | ap.AP_PROT_WRITE)
        ap.ap_bench_write(cache, r, ap.bench_cfg(ap.AP_UNIFORM, 4, 8, 256, reads_per_thread=8,
                                                 seed=3))
        # reads in a later kernel see the stores, written back or not
        out = torch.zeros(8 * 256, dtype=torch.int64, device="cuda")
        ap.ap_bench_read(cache, r, ap.bench_cfg(ap.AP_UNIFORM, 4, 8, 256, reads_per_thread=5,
                                                seed=99), out)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        assert np.array_equal(out.cpu().numpy().view(np.uint64),
                              oracle.read_uniform(want, n, 4, 8 * 256, 5, 99))
        ap.ap_munmap(cache, r)  # writes back whatever is still dirty
        assert np.array_equal(f, want)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("frames", [4, 200])
def test_apointer_copy_between_regions(ap, frames):
    """The paper's copy kernel with apointers on both sides."""
    n = (1 << 20) + 3 * 512
    src = make_file(n, seed=4)
    dst = make_file(n, seed=5)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        rs = ap.ap_mmap(cache, src)
        rd = ap.ap_mmap_prot(cache, dst, ap.AP_PROT_READ | ap.AP_PROT_WRITE)
        ap.ap_bench_copy(cache, rs, rd, ap.bench_cfg(ap.AP_SEQ, 16, 4, 128, unit_bytes=4096,
                                                     span_bytes=n))
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        assert check_invariants(ap, cache, [rs, rd], frames) == []
        ap.ap_munmap(cache, rd)
        ap.ap_munmap(cache, rs)
        assert np.array_equal(dst, src)
    finally:
        teardown(ap, cache)


def test_read_only_region_rejects_writes(ap):
    f = make_file(1 << 16, seed=6)
    cache = ap.ap_cache_create(8, 4096)
    try:
        r = ap.ap_mmap(cache, f)
        with pytest.raises(ap.APError):
            ap.ap_bench_write(cache, r, ap.bench_cfg(ap.AP_SEQ, 4, 1, 32, unit_bytes=4096))
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)
