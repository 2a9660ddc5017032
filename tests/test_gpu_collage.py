"""Parity of the collage kernel and the GPU-built LSH index against the oracle
(O3): bucket CSR bit-exact, winners (image index, squared
distance) bit-exact, for every candidate grouping, with the page cache smaller
than the dataset (eviction) and on the raw-pointer twin."""
import numpy as np
import pytest
import torch

import oracle
import synth
from helpers import check_invariants, make_records, teardown
from paper_conf_isca_shaharbs16_b200 import mgpu

pytestmark = pytest.mark.gpu


def _setup(n, W, H, L, K, w, bb, seed=21, stride=4096, frames=256, page=4096):  # noqa: ARG001
    recs = make_records(n, stride, seed)
    proj, bias = synth.make_lsh_params(L, K, w, seed=seed + 1)
    img, src, is_copy = synth.make_target(W, H, n, ds_seed=seed, seed=seed + 2, pool=32,
                                          copy_permille=100)
    return recs, proj, bias, img, src, is_copy


def _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev):
    L, K = bias.shape
    off = torch.zeros((L, (1 << bb) + 1), dtype=torch.int32, device=dev)
    ids = torch.zeros((L, n), dtype=torch.int32, device=dev)
    pd = torch.from_numpy(proj).to(dev)
    bd = torch.from_numpy(bias).to(dev)
    ap.ap_lsh_build_index(cache, r, n, stride, L, K, bb, w, pd, bd, off, ids)
    return off, ids, pd, bd


@pytest.mark.parametrize("K,bb", [(8, 10), (0, 4), (3, 6)])
def test_index_matches_oracle(ap, K, bb):
    dev = torch.device("cuda:0")
    n, stride, w = 3000, 4096, 2500
    recs, proj, bias, *_ = _setup(n, 64, 64, 4, K, w, bb)
    cache = ap.ap_cache_create(64, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off, ids, _, _ = _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev)
        want_off, want_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
        assert np.array_equal(off.cpu().numpy().view(np.uint32), want_off)
        assert np.array_equal(ids.cpu().numpy().view(np.uint32), want_ids)
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("group,schedule", [(1, 0), (1, 1), (2, 1), (4, 0), (4, 1), (8, 0), (8, 1), (1, 2), (8, 2), (1, 3), (8, 3),
                                            (16, 2), (32, 2), (32, 0)])
@pytest.mark.parametrize("frames", [48, 5000])
def test_collage_matches_oracle(ap, group, schedule, frames):
    dev = torch.device("cuda:0")
    n, stride, w, bb, L, K = 4096, 4096, 2500, 9, 4, 6
    W, H = 512, 256
    recs, proj, bias, img, src, is_copy = _setup(n, W, H, L, K, w, bb)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off, ids, pd, bd = _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev)
        tgt = torch.from_numpy(img).to(dev)
        nb = (W // 32) * (H // 32)
        win = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        inp = ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n, stride, group=group,
                            schedule=schedule)
        ap.ap_collage_run(cache, r, inp, win)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        got = win.cpu().numpy().view(np.uint32)
        # the oracle runs on its own index (never on the GPU-built CSR); the
        # GPU index must equal it bit for bit
        o_off, o_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
        assert np.array_equal(off.cpu().numpy().view(np.uint32), o_off)
        assert np.array_equal(ids.cpu().numpy().view(np.uint32), o_ids)
        want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, o_off, o_ids)
        assert np.array_equal(got, want)
        # planted copies found at distance 0
        assert np.all(got[is_copy.astype(bool), 1] == 0)
        assert check_invariants(ap, cache, [r], frames) == []
        # raw twin on a resident HBM copy of the file
        rawd = torch.from_numpy(recs).to(dev)
        win2 = torch.zeros_like(win)
        inp2 = ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n, stride, group=group,
                             mode=ap.AP_MODE_RAW, raw_base=rawd, schedule=schedule)
        ap.ap_collage_run(cache, r, inp2, win2)
        torch.cuda.synchronize()
        assert np.array_equal(win2.cpu().numpy().view(np.uint32), want)
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


def test_collage_partitioned_blocks_equal_whole(ap):
    """The multi-GPU partition on one GPU: block ranges run one
    after the other and concatenated equal the single run."""
    dev = torch.device("cuda:0")
    n, stride, w, bb = 2048, 4096, 2500, 8
    W, H = 256, 256
    recs, proj, bias, img, *_ = _setup(n, W, H, 2, 5, w, bb, seed=5)
    cache = ap.ap_cache_create(100, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off, ids, pd, bd = _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev)
        tgt = torch.from_numpy(img).to(dev)
        nb = (W // 32) * (H // 32)
        full = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n), full)
        parts = []
        for g in range(3):
            b0, b1 = g * nb // 3, (g + 1) * nb // 3
            part = torch.zeros((b1 - b0, 2), dtype=torch.int32, device=dev)
            ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n,
                                                      block_begin=b0, block_count=b1 - b0,
                                                      schedule=g % 3), part)
            parts.append(part)
        assert torch.equal(torch.cat(parts), full)
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("schedule", [2, 3])
@pytest.mark.parametrize("world", [2, 3, 8])
def test_collage_unit_slices_min_reduce_to_whole(ap, world, schedule):
    """The bucket partition (mgpu.unit_range + reduce_winners_min) on one GPU:
    each slice of the (table, bucket)-sorted units runs alone into its own
    winners array; the unsigned 64-bit MIN over the slices equals the single
    run and the oracle."""
    dev = torch.device("cuda:0")
    n, stride, w, bb, L, K = 2048, 4096, 2500, 8, 4, 5
    W, H = 256, 192
    recs, proj, bias, img, *_ = _setup(n, W, H, L, K, w, bb, seed=6)
    cache = ap.ap_cache_create(90, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off, ids, pd, bd = _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev)
        tgt = torch.from_numpy(img).to(dev)
        nb = (W // 32) * (H // 32)
        full = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n,
                                                  group=8), full)
        flip = torch.tensor(-(1 << 63), dtype=torch.int64, device=dev)
        acc = None
        for g in range(world):
            u0, u1 = mgpu.unit_range(L * nb, g, world)
            part = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
            ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n,
                                                      group=8, unit_begin=u0,
                                                      unit_count=u1 - u0, schedule=schedule),
                              part)
            f = part.view(torch.int64).view(-1) ^ flip
            acc = f if acc is None else torch.minimum(acc, f)
        got = (acc ^ flip).view(torch.int32).view(-1, 2)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        assert torch.equal(got, full)
        o_off, o_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
        want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, o_off, o_ids)
        assert np.array_equal(got.cpu().numpy().view(np.uint32), want)
        assert check_invariants(ap, cache, [r], 90) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("group,schedule", [(1, 1), (2, 1), (4, 1), (8, 1), (4, 2), (8, 2), (8, 3), (16, 2),
                                            (32, 2)])
@pytest.mark.parametrize("frames", [40, 3000])
def test_unaligned_records_collage(ap, group, schedule, frames):
    """NEXT N1: 3 KiB histograms without padding, so records
    straddle 4 KiB pages; the same kernel and pointers must still match the
    oracle bit for bit."""
    dev = torch.device("cuda:0")
    n, stride, w, bb, L, K = 4096, 3072, 2500, 9, 4, 6
    W, H = 384, 256
    recs, proj, bias, img, src, is_copy = _setup(n, W, H, L, K, w, bb, stride=stride)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off, ids, pd, bd = _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev)
        o_off, o_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
        assert np.array_equal(off.cpu().numpy().view(np.uint32), o_off)
        assert np.array_equal(ids.cpu().numpy().view(np.uint32), o_ids)
        tgt = torch.from_numpy(img).to(dev)
        nb = (W // 32) * (H // 32)
        win = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n, stride,
                                                  group=group, schedule=schedule), win)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, o_off, o_ids)
        assert np.array_equal(win.cpu().numpy().view(np.uint32), want)
        assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("schedule,chunks,frames", [(2, 2, 40), (2, 5, 40), (3, 3, 40), (3, 7, 400)])
def test_collage_record_id_windows(ap, schedule, chunks, frames):
    """ap_collage_in.id_chunks: the units run once per record-id window, each
    pass reading only candidates in its window; winners equal the one-pass
    run and the oracle, with a cache smaller and larger than the touched
    records, and also when the windows run over a slice of the units."""
    dev = torch.device("cuda:0")
    n, stride, w, bb, L, K = 2048, 4096, 2500, 8, 4, 5
    W, H = 256, 192
    recs, proj, bias, img, *_ = _setup(n, W, H, L, K, w, bb, seed=8)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off, ids, pd, bd = _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev)
        tgt = torch.from_numpy(img).to(dev)
        nb = (W // 32) * (H // 32)
        one = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n, group=8,
                                                  schedule=schedule), one)
        win = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_cache_reset(cache)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n, group=8,
                                                  schedule=schedule, id_chunks=chunks), win)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        assert torch.equal(win, one)
        o_off, o_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
        want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, o_off, o_ids)
        assert np.array_equal(win.cpu().numpy().view(np.uint32), want)
        # two unit slices, each with windows, MIN-combined
        flip = torch.tensor(-(1 << 63), dtype=torch.int64, device=dev)
        acc = None
        for g in range(2):
            u0, u1 = mgpu.unit_range(L * nb, g, 2)
            part = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
            ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n,
                                                      group=8, schedule=schedule, unit_begin=u0,
                                                      unit_count=u1 - u0, id_chunks=chunks), part)
            f = part.view(torch.int64).view(-1) ^ flip
            acc = f if acc is None else torch.minimum(acc, f)
        assert torch.equal((acc ^ flip).view(torch.int32).view(-1, 2), one)
        assert check_invariants(ap, cache, [r], frames) == []
        from paper_conf_isca_shaharbs16_b200._lib import APError
        with pytest.raises(APError):  # windows need per-table units
            ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n,
                                                      schedule=1, id_chunks=2), win)
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("world,chunks", [(2, 0), (3, 2), (8, 1)])
def test_collage_record_slices_min_reduce_to_whole(ap, world, chunks):
    """The by-records partition (mgpu.id_range + reduce_winners_min) on one
    GPU: each rank's record-id slice, all units, runs alone; the MIN over
    the slices equals the single run and the oracle; each slice fills only
    pages of its own records."""
    dev = torch.device("cuda:0")
    n, stride, w, bb, L, K = 2048, 4096, 2500, 8, 4, 5
    W, H = 256, 192
    recs, proj, bias, img, *_ = _setup(n, W, H, L, K, w, bb, seed=9)
    cache = ap.ap_cache_create(60, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off, ids, pd, bd = _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev)
        tgt = torch.from_numpy(img).to(dev)
        nb = (W // 32) * (H // 32)
        full = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n,
                                                  group=8), full)
        flip = torch.tensor(-(1 << 63), dtype=torch.int64, device=dev)
        acc = None
        for g in range(world):
            i0, i1 = mgpu.id_range(n, g, world)
            ap.ap_cache_reset(cache)
            part = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
            ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n,
                                                      group=8, id_chunks=chunks, id_begin=i0,
                                                      id_end=i1), part)
            torch.cuda.synchronize()
            # only this slice's record pages were ever filled
            pte = ap.ap_region_dump_pte(cache, r)
            touched = np.nonzero((pte >> np.uint64(62)) != 0)[0]
            assert touched.size == 0 or (touched.min() >= i0 and touched.max() < i1)
            f = part.view(torch.int64).view(-1) ^ flip
            acc = f if acc is None else torch.minimum(acc, f)
        got = (acc ^ flip).view(torch.int32).view(-1, 2)
        assert ap.ap_last_device_error(cache) == 0
        assert torch.equal(got, full)
        o_off, o_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
        want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, o_off, o_ids)
        assert np.array_equal(got.cpu().numpy().view(np.uint32), want)
        from paper_conf_isca_shaharbs16_b200._lib import APError
        for bad in (dict(id_begin=5, id_end=5), dict(id_begin=0, id_end=n + 1),
                    dict(id_begin=1, id_end=9, schedule=1)):
            with pytest.raises(APError):
                ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n,
                                                          **bad), part)
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("schedule", [0, 1, 2, 3])
@pytest.mark.parametrize("group", [1, 8])
def test_empty_candidate_sets_give_the_sentinel(ap, group, schedule):
    """R-A4: a block whose L buckets are all empty has no candidate; its
    winner is (0xFFFFFFFF, 0xFFFFFFFF).  A small dataset spread over 2^14
    buckets with one table leaves most blocks without candidates (planted
    copies still find theirs); every schedule must reproduce the oracle,
    sentinels included, from the oracle's own index."""
    dev = torch.device("cuda:0")
    n, stride, w, bb, L, K = 512, 4096, 2500, 14, 1, 8
    W, H = 256, 256
    recs, proj, bias, img, src, is_copy = _setup(n, W, H, L, K, w, bb, seed=41)
    o_off, o_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
    want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, o_off, o_ids)
    empty = np.all(want == oracle.EMPTY, axis=1)
    assert empty.sum() > 0 and (~empty).sum() > 0, (empty.sum(), len(empty))
    cache = ap.ap_cache_create(32, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off, ids, pd, bd = _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev)
        assert np.array_equal(off.cpu().numpy().view(np.uint32), o_off)
        assert np.array_equal(ids.cpu().numpy().view(np.uint32), o_ids)
        tgt = torch.from_numpy(img).to(dev)
        nb = (W // 32) * (H // 32)
        win = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n, stride,
                                                  group=group, schedule=schedule), win)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        assert np.array_equal(win.cpu().numpy().view(np.uint32), want)
        assert check_invariants(ap, cache, [r], 32) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


@pytest.mark.parametrize("group", [4, 8])
@pytest.mark.parametrize("stride,frames", [(4096, 64), (4096, 5000), (3072, 40)])
def test_collage_warp_items_many_windows(ap, group, stride, frames):
    """A step with >= 2^20 (window, unit) items runs one warp per item
    (k_collage_wunit, with the precomputed window bounds and the empty-window
    exit): 1024 blocks x 4 tables x 256 windows.  Winners equal the one-pass
    run and the oracle (on its own index), with a cache smaller and larger
    than the touched records and with records straddling pages."""
    dev = torch.device("cuda:0")
    n, w, bb, L, K = 4096, 2500, 8, 4, 5
    W, H = 1024, 1024
    recs, proj, bias, img, *_ = _setup(n, W, H, L, K, w, bb, seed=12, stride=stride)
    cache = ap.ap_cache_create(frames, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off, ids, pd, bd = _gpu_index(ap, cache, r, n, stride, proj, bias, w, bb, dev)
        tgt = torch.from_numpy(img).to(dev)
        nb = (W // 32) * (H // 32)
        one = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n, stride,
                                                  group=group, schedule=2), one)
        win = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_cache_reset(cache)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n, stride,
                                                  group=group, schedule=2, id_chunks=256), win)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        assert torch.equal(win, one)
        o_off, o_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
        want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, o_off, o_ids)
        assert np.array_equal(win.cpu().numpy().view(np.uint32), want)
        assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)
