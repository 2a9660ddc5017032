"""Parity of apointer reads (CUDA path through the C ABI) against the oracle
(O1: plain file indexing) and the page-cache invariants (O2), across cache
sizes, eviction policies, patterns and element sizes.  Every value must be
bit-exact: faults and eviction order are invisible to values (PAPER.md:121,
141-145)."""
import numpy as np
import pytest
import torch

import oracle
from helpers import check_invariants, make_file, teardown

pytestmark = pytest.mark.gpu


@pytest.fixture
def dev():
    assert torch.cuda.is_available(), "GPU tests need a B200"
    return torch.device("cuda:0")


def _run(ap, cache, region, cfg, nthreads, dev, out_bytes=None):
    out = torch.zeros(out_bytes if out_bytes else nthreads * 8, dtype=torch.uint8, device=dev)
    ap.ap_bench_read(cache, region, cfg, out)
    torch.cuda.synchronize()
    assert ap.ap_last_device_error(cache) == 0
    return out.cpu().numpy()


import os

# AP_ACCESS_TILE, _RANGE, _AHEAD, _PAIR; the split-phase styles (AHEAD, PAIR)
# are not part of the hash-table ablation build
ACCESS = [0, 2] if "hash" in os.environ.get("AP_LIB_PATH", "") else [0, 2, 3, 4]


@pytest.mark.parametrize("access", ACCESS)
@pytest.mark.parametrize("frames", [1, 8, 64, 4096])
@pytest.mark.parametrize("elem", [4, 16])
def test_seq_copy_is_the_file(ap, dev, frames, elem, access):
    """C1 shape: warps walk pages, every read faults while frames < pages.
    Both tiled access styles (tiles; one pin per unit) give the file."""
    nbytes = (1 << 20) + 3 * 4096 + 48  # ragged last page
    f = make_file(nbytes, seed=1)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        r = ap.ap_mmap(cache, f)
        grid, block = (2, 64) if frames == 1 else (8, 128)
        cfg = ap.bench_cfg(ap.AP_SEQ, elem, grid, block, unit_bytes=4096, out_copy=True,
                           span_bytes=nbytes, access=access)
        out = _run(ap, cache, r, cfg, grid * block, dev, out_bytes=nbytes)
        whole = nbytes // elem * elem
        assert np.array_equal(out[:whole], f[:whole])
        assert check_invariants(ap, cache, [r], frames) == []
        st = ap.ap_cache_stats(cache)
        npages = (nbytes + 4095) // 4096
        if frames >= npages:
            assert st["major"] == npages and st["evictions"] == 0
        else:
            assert st["major"] >= npages and st["evictions"] >= npages - frames
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("policy", ["clock", "sequential"])
@pytest.mark.parametrize("frames", [1, 3, 64, 4096])
@pytest.mark.parametrize("mode", ["apointer", "raw"])
def test_seq_queue_copy_is_the_file(ap, dev, frames, policy, mode):
    """AP_SEQ_QUEUE (units handed out from a device counter, the C1 launch):
    whichever warp reads a unit, every byte lands at its offset -- the file,
    ragged tail included -- invariants hold, and 2 units per warp or fewer
    than one unit per warp both work.  Its twin reads the zero-copy host
    bytes through the same queue."""
    nbytes = (1 << 20) + 3 * 4096 + 48
    f = make_file(nbytes, seed=7)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        ap.ap_cache_set_policy(cache, ap.AP_POLICY_SEQUENTIAL if policy == "sequential"
                               else ap.AP_POLICY_CLOCK)
        r = ap.ap_mmap(cache, f)
        for grid, block in ((2, 64), (148, 32), (300, 32)):
            if frames == 1 and grid * block > 64:
                continue
            kw = dict(mode=ap.AP_MODE_RAW, raw_base=ap.ap_region_devptr(cache, r)) \
                if mode == "raw" else {}
            cfg = ap.bench_cfg(ap.AP_SEQ_QUEUE, 16, grid, block, unit_bytes=4096,
                               out_copy=True, span_bytes=nbytes, **kw)
            for rep in range(2):  # the counter restarts at every launch
                out = _run(ap, cache, r, cfg, grid * block, dev, out_bytes=nbytes)
                assert np.array_equal(out[:nbytes // 16 * 16], f[:nbytes // 16 * 16]), (grid, rep)
        assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


def test_stats_live_refcnt_sum_and_err(ap, dev):
    """SURVEY B5's counters: live_refcnt_sum is the page tables' reference
    counts (0 once every apointer is gone; equal to the sum over
    the PTE dump), backoff_spins = waits, err = the sticky error word (read
    without clearing it)."""
    nbytes = (1 << 21) + 4096 + 48
    f = make_file(nbytes, seed=9)
    cache = ap.ap_cache_create(8, 4096)
    try:
        r = ap.ap_mmap(cache, f)
        cfgs = [ap.bench_cfg(ap.AP_SEQ_QUEUE, 16, 20, 32, unit_bytes=4096, out_copy=True,
                             span_bytes=nbytes),
                ap.bench_cfg(ap.AP_UNIFORM, 4, 6, 128, reads_per_thread=5, seed=3),
                ap.bench_cfg(ap.AP_DIVERGENT, 4, 4, 64, reads_per_thread=3, page_bytes=4096,
                             seed=5)]
        for cfg in cfgs:
            out = torch.zeros(max(nbytes, 20 * 32 * 8), dtype=torch.uint8, device=dev)
            ap.ap_bench_read(cache, r, cfg, out)
            st = ap.ap_cache_stats(cache)
            rc = (ap.ap_region_dump_pte(cache, r) & np.uint64(0xffffffff)).sum()
            assert st["live_refcnt_sum"] == int(rc) == 0
            assert st["err"] == 0 and st["backoff_spins"] == st["waits"]
            assert ap.ap_last_device_error(cache) == 0
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


def test_seq_queue_rejects_checksums_and_other_access(ap, dev):
    """The queue's unit order is dynamic, so per-thread checksums (which
    depend on which units a thread read) and the other access styles are
    refused."""
    from paper_conf_isca_shaharbs16_b200._lib import APError
    f = make_file(1 << 20, seed=8)
    cache = ap.ap_cache_create(64, 4096)
    try:
        r = ap.ap_mmap(cache, f)
        out = torch.zeros(1 << 20, dtype=torch.uint8, device=dev)
        for kw in (dict(out_copy=False), dict(out_copy=True, access=ap.AP_ACCESS_RANGE)):
            cfg = ap.bench_cfg(ap.AP_SEQ_QUEUE, 16, 4, 64, unit_bytes=4096, **kw)
            with pytest.raises(APError):
                ap.ap_bench_read(cache, r, cfg, out)
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("elem,unit,passes", [(16, 4096, 1), (16, 16384, 3), (4, 2048, 2),
                                              (8, 65536, 1)])
@pytest.mark.parametrize("access", ACCESS)
def test_seq_checksums(ap, dev, elem, unit, passes, access):
    page = 65536
    nbytes = 4 * (1 << 20) + 777 * 16
    f = make_file(nbytes, seed=2)
    cache = ap.ap_cache_create(32, page)
    try:
        r = ap.ap_mmap(cache, f)
        grid, block = 6, 256
        cfg = ap.bench_cfg(ap.AP_SEQ, elem, grid, block, unit_bytes=unit, passes=passes,
                           span_bytes=nbytes, access=access)
        got = _run(ap, cache, r, cfg, grid * block, dev).view(np.uint64)
        want = oracle.read_seq(f, nbytes, unit, elem, grid * block, passes)
        assert np.array_equal(got, want)
        assert check_invariants(ap, cache, [r], 32) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("policy,seed", [(0, 0), (1, 1), (1, 2), (1, 3)])
@pytest.mark.parametrize("frames", [3, 64, 2048])
def test_uniform_random_any_eviction_order(ap, dev, policy, seed, frames):
    page, nbytes = 4096, 4 << 20
    f = make_file(nbytes, seed=3)
    cache = ap.ap_cache_create(frames, page)
    try:
        ap.ap_cache_set_policy(cache, policy, seed)
        r = ap.ap_mmap(cache, f)
        grid, block, reads = 12, 128, 6
        cfg = ap.bench_cfg(ap.AP_UNIFORM, 4, grid, block, reads_per_thread=reads, seed=99)
        got = _run(ap, cache, r, cfg, grid * block, dev).view(np.uint64)
        want = oracle.read_uniform(f, nbytes, 4, grid * block, reads, 99)
        assert np.array_equal(got, want)
        assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("elem,page,frames", [(4, 4096, 256), (16, 4096, 40), (4, 65536, 64)])
def test_divergent_distinct_pages(ap, dev, elem, page, frames):
    nbytes = 200 * page
    f = make_file(nbytes, seed=4)
    cache = ap.ap_cache_create(frames, page)
    try:
        r = ap.ap_mmap(cache, f)
        grid, block, reads = 8, 256, 4
        cfg = ap.bench_cfg(ap.AP_DIVERGENT, elem, grid, block, reads_per_thread=reads,
                           page_bytes=page, seed=5)
        got = _run(ap, cache, r, cfg, grid * block, dev).view(np.uint64)
        want = oracle.read_divergent(f, nbytes, page, elem, grid * block, reads, 5)
        assert np.array_equal(got, want)
        assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


def test_hit_mode_after_prefill_has_no_major_faults(ap, dev):
    page, nbytes, frames = 65536, 64 << 20, 1024
    f = make_file(nbytes, seed=6)
    cache = ap.ap_cache_create(frames, page)
    try:
        r = ap.ap_mmap(cache, f)
        ap.ap_prefill(cache, r, 0, nbytes // page)
        torch.cuda.synchronize()
        st0 = ap.ap_cache_stats(cache)
        assert st0["major"] == nbytes // page
        grid, block = 148, 512
        cfg = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=16384, passes=2)
        got = _run(ap, cache, r, cfg, grid * block, dev).view(np.uint64)
        want = oracle.read_seq(f, nbytes, 16384, 16, grid * block, 2)
        assert np.array_equal(got, want)
        st1 = ap.ap_cache_stats(cache)
        assert st1["major"] == st0["major"]
        # SEQ with unit | page, all lanes of a warp on one page, one pointer per
        # thread walking its units: one link each time the warp's next unit is
        # on another page than the one it holds -- a warp whose
        # only unit is revisited by the next pass keeps its link
        W, nunits, upp = grid * block // 32, nbytes // 16384, page // 16384
        links = 0
        for w in range(W):
            pages = [u // upp for _ in range(2) for u in range(w, nunits, W)]
            links += sum(1 for i, p in enumerate(pages) if i == 0 or p != pages[i - 1])
        assert st1["minor"] - st0["minor"] == links
        assert check_invariants(ap, cache, [r], frames) == []
        # raw twin over an HBM copy reads the same values
        dcopy = torch.from_numpy(f).to(dev)
        cfg_raw = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=16384, passes=2,
                               mode=ap.AP_MODE_RAW, raw_base=dcopy.data_ptr())
        raw = _run(ap, cache, r, cfg_raw, grid * block, dev).view(np.uint64)
        assert np.array_equal(raw, want)
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


def test_zero_copy_raw_twin_uniform(ap, dev):
    nbytes = 8 << 20
    f = make_file(nbytes, seed=7)
    cache = ap.ap_cache_create(16, 65536)
    try:
        r = ap.ap_mmap(cache, f)
        base = ap.ap_region_devptr(cache, r)
        cfg = ap.bench_cfg(ap.AP_UNIFORM, 4, 16, 256, reads_per_thread=3, seed=11,
                           mode=ap.AP_MODE_RAW, raw_base=base)
        got = _run(ap, cache, r, cfg, 16 * 256, dev).view(np.uint64)
        assert np.array_equal(got, oracle.read_uniform(f, nbytes, 4, 16 * 256, 3, 11))
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


def test_two_regions_share_one_cache(ap, dev):
    f1, f2 = make_file(3 << 20, seed=8), make_file(5 << 20, seed=9)
    cache = ap.ap_cache_create(50, 4096)
    try:
        r1, r2 = ap.ap_mmap(cache, f1), ap.ap_mmap(cache, f2)
        for r, f in ((r1, f1), (r2, f2), (r1, f1)):
            cfg = ap.bench_cfg(ap.AP_UNIFORM, 4, 4, 256, reads_per_thread=4, seed=3)
            got = _run(ap, cache, r, cfg, 1024, dev).view(np.uint64)
            assert np.array_equal(got, oracle.read_uniform(f, f.nbytes, 4, 1024, 4, 3))
        assert check_invariants(ap, cache, [r1, r2], 50) == []
        ap.ap_munmap(cache, r1)
        assert check_invariants(ap, cache, [r2], 50) == []
        ap.ap_munmap(cache, r2)
    finally:
        teardown(ap, cache)


def test_reset_starts_cold(ap, dev):
    f = make_file(2 << 20, seed=10)
    cache = ap.ap_cache_create(600, 4096)
    try:
        r = ap.ap_mmap(cache, f)
        cfg = ap.bench_cfg(ap.AP_SEQ, 16, 4, 128, unit_bytes=4096)
        for _ in range(2):
            ap.ap_cache_reset(cache)
            _run(ap, cache, r, cfg, 512, dev)
            st = ap.ap_cache_stats(cache)
            assert st["major"] == 512 and st["evictions"] == 0
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("elem", [4, 16])
def test_uniform_over_resident_span_minor_faults(ap, dev, elem):
    """M2r: offsets uniform over a resident span (span_bytes < region), every
    read a minor fault through the inline link path; values == oracle over
    the span, no major faults, one link per (warp, distinct page) group."""
    page, nbytes, span = 65536, 32 << 20, 8 << 20
    f = make_file(nbytes, seed=12)
    cache = ap.ap_cache_create(span // page + 8, page)
    try:
        r = ap.ap_mmap(cache, f)
        ap.ap_prefill(cache, r, 0, span // page)
        torch.cuda.synchronize()
        st0 = ap.ap_cache_stats(cache)
        grid, block, reads = 296, 512, 5
        cfg = ap.bench_cfg(ap.AP_UNIFORM, elem, grid, block, reads_per_thread=reads, seed=21,
                           span_bytes=span)
        got = _run(ap, cache, r, cfg, grid * block, dev).view(np.uint64)
        want = oracle.read_uniform(f[:span], span, elem, grid * block, reads, 21)
        assert np.array_equal(got, want)
        st1 = ap.ap_cache_stats(cache)
        assert st1["major"] == st0["major"]
        assert st1["minor"] > st0["minor"]
        assert check_invariants(ap, cache, [r], span // page + 8) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("frames", [3, 512])
def test_per_access_deref_kernel(ap, dev, frames):
    """The per-access `v = *q; q += 32` kernel (full-occupancy build) and its
    raw per-access twin both equal the oracle, with the cache smaller and
    larger than the span."""
    page, nbytes = 4096, 1 << 20
    f = make_file(nbytes, seed=13)
    cache = ap.ap_cache_create(frames, page)
    try:
        r = ap.ap_mmap(cache, f)
        grid, block = 16, 512
        cfg = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=4096, passes=2,
                           access=ap.AP_ACCESS_DEREF)
        got = _run(ap, cache, r, cfg, grid * block, dev).view(np.uint64)
        want = oracle.read_seq(f, nbytes, 4096, 16, grid * block, 2)
        assert np.array_equal(got, want)
        dcopy = torch.from_numpy(f).to(dev)
        cfg_raw = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=4096, passes=2,
                               access=ap.AP_ACCESS_DEREF, mode=ap.AP_MODE_RAW,
                               raw_base=dcopy.data_ptr())
        assert np.array_equal(_run(ap, cache, r, cfg_raw, grid * block, dev).view(np.uint64), want)
        assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("prefill,frames,unit", [(True, 1024, 65536), (False, 24, 16384),
                                                 (False, 3, 65536)])
def test_seq_tma_staged(ap, dev, prefill, frames, unit):
    """AP_ACCESS_TMA: the SEQ stream staged through shared memory by TMA bulk
    copies, one pin per unit; apointer and raw twin == oracle, resident or
    faulting (3 frames: every unit evicts, two units pinned per warp at most).
    A launch whose resident warps could pin more than the frames (two units
    per warp) is refused instead of waiting into the watchdog."""
    page, nbytes = 65536, 16 << 20
    f = make_file(nbytes, seed=41)
    cache = ap.ap_cache_create(frames, page)
    try:
        r = ap.ap_mmap(cache, f)
        if prefill:
            ap.ap_prefill(cache, r, 0, min(frames, nbytes // page))
            torch.cuda.synchronize()
        grid, block = {1024: (148, 512), 24: (1, 256), 3: (1, 32)}[frames]
        cfg = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=unit, passes=2,
                           access=ap.AP_ACCESS_TMA)
        got = _run(ap, cache, r, cfg, grid * block, dev).view(np.uint64)
        want = oracle.read_seq(f, nbytes, unit, 16, grid * block, 2)
        assert np.array_equal(got, want)
        dcopy = torch.from_numpy(f).to(dev)
        cfg_raw = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=unit, passes=2,
                               access=ap.AP_ACCESS_TMA, mode=ap.AP_MODE_RAW,
                               raw_base=dcopy.data_ptr())
        assert np.array_equal(_run(ap, cache, r, cfg_raw, grid * block, dev).view(np.uint64), want)
        assert check_invariants(ap, cache, [r], frames) == []
        from paper_conf_isca_shaharbs16_b200._lib import APError
        if frames < min(2 * 148 * 16, nbytes // page):
            with pytest.raises(APError):  # too few frames for 2 pins per resident warp
                ap.ap_bench_read(cache, r, ap.bench_cfg(ap.AP_SEQ, 16, 148, 512, unit_bytes=unit,
                                                        access=ap.AP_ACCESS_TMA),
                                 torch.zeros(148 * 512, dtype=torch.int64, device=dev))
        with pytest.raises(APError):  # 4-B elements are not staged
            ap.ap_bench_read(cache, r, ap.bench_cfg(ap.AP_SEQ, 4, 1, 32, unit_bytes=unit,
                                                    access=ap.AP_ACCESS_TMA),
                             torch.zeros(32, dtype=torch.int64, device=dev))
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("pattern,elem,page,nbytes,prefill", [
    (2, 4, 4096, 256 << 20, False),   # C3 shape, cold: every link a major fault
    (2, 16, 4096, 256 << 20, True),   # resident: every link a minor fault
    (2, 4, 65536, 512 << 20, False),
    (1, 4, 65536, 64 << 20, True),    # UNIFORM: lanes of a warp may share pages
    (1, 16, 4096, 16 << 20, True),
])
def test_link_events_closed_form(ap, dev, pattern, elem, page, nbytes, prefill):
    """O2 closed form: with a cache that
    never runs out of frames, major + minor faults == the number of (warp,
    iteration, distinct page) link events computed from the access trace
    alone (oracle.invariants.link_events) -- one leader per page per warp,
    DIVERGENT warps (32 distinct pages) and UNIFORM warps (shared pages)."""
    from oracle import invariants
    f = make_file(nbytes, seed=31)
    npages = nbytes // page
    frames = npages + 8  # never under frame pressure: no downgrade, no eviction
    cache = ap.ap_cache_create(frames, page)
    try:
        r = ap.ap_mmap(cache, f)
        if prefill:
            ap.ap_prefill(cache, r, 0, npages)
            torch.cuda.synchronize()
        grid, block, reads, seed = 32, 256, 4, 77
        nthreads = grid * block
        offs = oracle.offsets(pattern, nbytes, elem, nthreads, reads, seed, page)
        pg = offs >> np.uint64(page.bit_length() - 1)
        if not prefill:
            # cold runs wait on pages other warps are loading, and a waiting
            # warp may drop links it already holds (R-A19); that can only add
            # a link when a thread's next read is on the same page, which this
            # seeded trace never does
            assert not np.any(pg[:, 1:] == pg[:, :-1])
        want_links = invariants.link_events(offs, page.bit_length() - 1)
        st0 = ap.ap_cache_stats(cache)
        cfg = ap.bench_cfg(pattern, elem, grid, block, reads_per_thread=reads, seed=seed,
                           page_bytes=page if pattern == 2 else 0)
        got = _run(ap, cache, r, cfg, nthreads, dev).view(np.uint64)
        if pattern == 2:
            want = oracle.read_divergent(f, nbytes, page, elem, nthreads, reads, seed)
        else:
            want = oracle.read_uniform(f, nbytes, elem, nthreads, reads, seed)
        assert np.array_equal(got, want)
        st1 = ap.ap_cache_stats(cache)
        assert invariants.check_link_count(st0, st1, want_links) == []
        if prefill:
            assert st1["major"] == st0["major"]
        else:
            assert st1["major"] - st0["major"] == len(np.unique(pg))  # exactly once per page
        assert st1["evictions"] == 0
        assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("frames", [1, 3, 64, 4096])
@pytest.mark.parametrize("pattern", ["seq", "uniform"])
def test_sequential_policy_drop_behind(ap, dev, frames, pattern):
    """AP_POLICY_SEQUENTIAL (the clock + drop-behind: a faulting warp first
    reuses the frame of the page it just left): values are the file's bytes
    under any order of eviction, invariants hold, and a
    single-pass stream through few frames recycles frames without sweeping."""
    nbytes = (1 << 20) + 5 * 4096 + 32
    f = make_file(nbytes, seed=91)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        ap.ap_cache_set_policy(cache, ap.AP_POLICY_SEQUENTIAL)
        r = ap.ap_mmap(cache, f)
        if pattern == "seq":
            grid, block = (2, 64) if frames < 8 else (8, 128)
            cfg = ap.bench_cfg(ap.AP_SEQ, 16, grid, block, unit_bytes=4096, out_copy=True,
                               span_bytes=nbytes)
            out = _run(ap, cache, r, cfg, grid * block, dev, out_bytes=nbytes)
            whole = nbytes // 16 * 16
            assert np.array_equal(out[:whole], f[:whole])
        else:
            grid, block, reads = 6, 128, 5
            cfg = ap.bench_cfg(ap.AP_UNIFORM, 4, grid, block, reads_per_thread=reads, seed=19)
            got = _run(ap, cache, r, cfg, grid * block, dev).view(np.uint64)
            assert np.array_equal(got, oracle.read_uniform(f, nbytes, 4, grid * block, reads, 19))
        assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)
