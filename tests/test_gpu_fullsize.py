"""Parity at BASELINE.json's full sizes, in the launch configurations bench.py
times: C1, C2 and C3 read sets and the C4 collage, every
output compared with the oracle (O1 / O3) -- the read checksums and the
collage winners of every block -- plus the page-cache invariants (O2).
C5 (a 40 GB file) is checked on sampled blocks by bench.py itself."""
import numpy as np
import pytest
import torch

import oracle
import synth
from helpers import aligned_empty, check_invariants, make_file, teardown

pytestmark = pytest.mark.gpu

GiB = 1 << 30


@pytest.fixture(scope="module")
def dev():
    assert torch.cuda.is_available(), "GPU tests need a B200"
    return torch.device("cuda:0")


def _read(ap, cache, r, cfg, n):
    out = torch.zeros(n, dtype=torch.int64, device="cuda")
    ap.ap_bench_read(cache, r, cfg, out)
    torch.cuda.synchronize()
    assert ap.ap_last_device_error(cache) == 0
    return out.cpu().numpy().view(np.uint64)


def test_c1_full_copy(ap, dev):
    """C1: 16 MiB file, 4 KiB pages, 64 frames, 148 warps, 16-B SEQ copy."""
    f = make_file(16 << 20, 1)
    cache = ap.ap_cache_create(64, 4096)
    try:
        r = ap.ap_mmap(cache, f)
        out = torch.zeros(16 << 20, dtype=torch.uint8, device=dev)
        cfg = ap.bench_cfg(ap.AP_SEQ, 16, 148, 32, unit_bytes=4096, out_copy=True)
        ap.ap_bench_read(cache, r, cfg, out)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        assert np.array_equal(out.cpu().numpy(), f)
        st = ap.ap_cache_stats(cache)
        assert st["major"] == 4096  # every page once (SEQ, one warp per page)
        assert check_invariants(ap, cache, [r], 64) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


def test_c2_full(ap, dev):
    """C2: 4 GiB file, 64 KiB pages, 1 GiB cache, uniform 4-B reads, 148 x 512
    threads, 8 reads each (the bench's launch); every checksum == oracle."""
    f = make_file(4 * GiB, 1)
    cache = ap.ap_cache_create(16384, 65536)
    try:
        r = ap.ap_mmap(cache, f)
        n = 148 * 512
        cfg = ap.bench_cfg(ap.AP_UNIFORM, 4, 148, 512, reads_per_thread=8, seed=1234)
        got = _read(ap, cache, r, cfg, n)
        assert np.array_equal(got, oracle.read_uniform(f, 4 * GiB, 4, n, 8, 1234))
        st = ap.ap_cache_stats(cache)
        assert st["evictions"] > 0  # the cache is a quarter of the file
        assert check_invariants(ap, cache, [r], 16384) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)


def test_c3_full(ap, dev):
    """C3: 16 GiB file, 4 KiB pages, 256 MiB cache, 32 lanes of a warp on 32
    distinct pages, 4-B reads, 148 x 512 threads, 4 reads each."""
    f = make_file(16 * GiB, 1)
    cache = ap.ap_cache_create(65536, 4096)
    try:
        r = ap.ap_mmap(cache, f)
        n = 148 * 512
        cfg = ap.bench_cfg(ap.AP_DIVERGENT, 4, 148, 512, reads_per_thread=4, page_bytes=4096,
                           seed=77)
        got = _read(ap, cache, r, cfg, n)
        assert np.array_equal(got, oracle.read_divergent(f, 16 * GiB, 4096, 4, n, 4, 77))
        assert check_invariants(ap, cache, [r], 65536) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)
    del f


@pytest.mark.parametrize("schedule", [2, 1, 3])
def test_c4_full(ap, dev, schedule):
    """C4: 1M records (4 GiB), 1024x1024 target, L=4 K=8 2^14 buckets, 256 MiB
    cache, 8 candidates per warp: the GPU-built index and the winners of all
    1024 blocks == oracle; planted copies find distance 0."""
    N, W, H, L, K, bb, w = 1 << 20, 1024, 1024, 4, 8, 14, 60000
    recs = synth.fill_records(aligned_empty(N * 4096), 0, N, 4096, 21)
    img, src, is_copy = synth.make_target(W, H, N, ds_seed=21, seed=23, pool=256,
                                          copy_permille=50)
    proj, bias = synth.make_lsh_params(L, K, w, seed=22)
    cache = ap.ap_cache_create(65536, 4096)
    try:
        r = ap.ap_mmap(cache, recs)
        off = torch.empty((L, (1 << bb) + 1), dtype=torch.int32, device=dev)
        ids = torch.empty((L, N), dtype=torch.int32, device=dev)
        pd, bd = torch.from_numpy(proj).to(dev), torch.from_numpy(bias).to(dev)
        ap.ap_lsh_build_index(cache, r, N, 4096, L, K, bb, w, pd, bd, off, ids)
        o_off, o_ids = oracle.build_index(recs, 4096, N, proj, bias, w, bb)
        assert np.array_equal(off.cpu().numpy().view(np.uint32), o_off)
        assert np.array_equal(ids.cpu().numpy().view(np.uint32), o_ids)
        tgt = torch.from_numpy(img).to(dev)
        nb = (W // 32) * (H // 32)
        win = torch.empty((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, N,
                                                  group=8, schedule=schedule), win)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        got = win.cpu().numpy().view(np.uint32)
        want = oracle.collage(img, proj, bias, w, bb, recs, 4096, N, o_off, o_ids)
        assert np.array_equal(got, want)
        planted = np.flatnonzero(np.asarray(is_copy).reshape(-1) != 0)
        assert planted.size > 0 and (got[planted, 1] == 0).all()
        assert check_invariants(ap, cache, [r], 65536) == []
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)
