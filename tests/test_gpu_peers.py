"""N2 peer page caches (PAPER.md:33 distributed shared memory
across GPUs): a major fault first copies the page from a peer cache that
holds it, else fills from the host.  Values must stay bit-exact against the
oracle (O1: plain file indexing) whichever source served a page, the peer
must keep its reference counts (its pages are pinned only during a copy),
and the fill accounting must split exactly between the two sources.

On one GPU the "peer" is a second cache on the same device (same-process
API) or in a second process (CUDA IPC); across GPUs the same code reads the
peer's HBM over NVLink."""
import multiprocessing as mp
import os

import numpy as np
import pytest
import torch

import oracle
from helpers import check_invariants, make_file, teardown

pytestmark = pytest.mark.gpu

PAGE = 65536


@pytest.fixture
def dev():
    assert torch.cuda.is_available(), "GPU tests need a B200"
    return torch.device("cuda:0")


def _copy(ap, cache, region, nbytes, dev, stream=None, grid=16, block=256, elem=16):
    cfg = ap.bench_cfg(ap.AP_SEQ, elem, grid, block, unit_bytes=PAGE, out_copy=True,
                       span_bytes=nbytes)
    out = torch.zeros(nbytes, dtype=torch.uint8, device=dev)
    ap.ap_bench_read(cache, region, cfg, out, stream)
    return out


def test_all_pages_from_a_full_peer(ap, dev):
    """Peer A holds every page: B's fills all come from A, none from the host."""
    nbytes = 8 * (1 << 20) + 3 * 4096 + 80  # ragged last page
    npages = (nbytes + PAGE - 1) // PAGE
    f = make_file(nbytes, seed=31)
    a = ap.ap_cache_create(npages, PAGE)
    b = ap.ap_cache_create(npages, PAGE)
    try:
        ra = ap.ap_mmap(a, f)
        rb = ap.ap_mmap(b, f)
        ap.ap_prefill(a, ra, 0, npages)
        torch.cuda.synchronize()
        sa0 = ap.ap_cache_stats(a)
        ap.ap_region_add_peer(b, rb, a, ra)
        out = _copy(ap, b, rb, nbytes, dev)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(b) == 0
        whole = nbytes // 16 * 16
        assert np.array_equal(out.cpu().numpy()[:whole], f[:whole])
        st = ap.ap_cache_stats(b)
        assert st["major"] == npages and st["peer_fills"] == npages
        assert st["fill_bytes"] == 0 and st["peer_bytes"] == npages * PAGE
        # A served the copies without faults of its own and holds no pins
        sa1 = ap.ap_cache_stats(a)
        assert sa1["major"] == sa0["major"] and sa1["evictions"] == 0
        assert check_invariants(ap, a, [ra], npages) == []
        assert check_invariants(ap, b, [rb], npages) == []
        # the ragged last page arrived zero-padded, as a host fill leaves it
        ap.ap_region_clear_peers(b, rb)
        ap.ap_munmap(b, rb)
        ap.ap_munmap(a, ra)
    finally:
        teardown(ap, b)
        teardown(ap, a)


def test_split_between_peer_and_host(ap, dev):
    """A holds the first half: B gets exactly that half from A and the rest
    over the host link, each page exactly once (B's cache >= the file)."""
    npages = 96
    nbytes = npages * PAGE - 4096 + 48
    f = make_file(nbytes, seed=32)
    a = ap.ap_cache_create(npages, PAGE)
    b = ap.ap_cache_create(npages, PAGE)
    try:
        ra = ap.ap_mmap(a, f)
        rb = ap.ap_mmap(b, f)
        half = npages // 2
        ap.ap_prefill(a, ra, 0, half)
        torch.cuda.synchronize()
        ap.ap_region_add_peer(b, rb, a, ra)
        out = _copy(ap, b, rb, nbytes, dev)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(b) == 0
        whole = nbytes // 16 * 16
        assert np.array_equal(out.cpu().numpy()[:whole], f[:whole])
        st = ap.ap_cache_stats(b)
        assert st["major"] == npages
        assert st["peer_fills"] == half
        assert st["fill_bytes"] == nbytes - half * PAGE
        assert check_invariants(ap, a, [ra], npages) == []
        assert check_invariants(ap, b, [rb], npages) == []
        ap.ap_munmap(b, rb)  # clears the peer list itself
        ap.ap_munmap(a, ra)
    finally:
        teardown(ap, b)
        teardown(ap, a)


@pytest.mark.parametrize("frames", [4, 48])
def test_mutual_peers_running_concurrently(ap, dev, frames):
    """A and B are each other's peer, both caches are smaller than the file
    and both run uniform-random reads at the same time on two streams: each
    evicts while the other pins its pages for copies.  Values == oracle on
    both sides, no pins left, and no deadlock (a peer copy never waits)."""
    npages = 64
    nbytes = npages * PAGE
    f = make_file(nbytes, seed=33)
    a = ap.ap_cache_create(frames, PAGE)
    b = ap.ap_cache_create(frames, PAGE)
    try:
        ra = ap.ap_mmap(a, f)
        rb = ap.ap_mmap(b, f)
        ap.ap_region_add_peer(a, ra, b, rb)
        ap.ap_region_add_peer(b, rb, a, ra)
        grid, block, reads = 32, 256, 6
        sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
        outs = {}
        for i in range(3):
            for cache, reg, s, seed in ((a, ra, sa, 40 + i), (b, rb, sb, 50 + i)):
                cfg = ap.bench_cfg(ap.AP_UNIFORM, 4, grid, block, reads_per_thread=reads,
                                   seed=seed)
                o = torch.zeros(grid * block * 8, dtype=torch.uint8, device=dev)
                ap.ap_bench_read(cache, reg, cfg, o, s)
                outs[seed] = o
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(a) == 0 and ap.ap_last_device_error(b) == 0
        for seed, o in outs.items():
            want = oracle.read_uniform(f, nbytes, 4, grid * block, reads, seed)
            assert np.array_equal(o.cpu().numpy().view(np.uint64), want), seed
        stt = [ap.ap_cache_stats(x) for x in (a, b)]
        assert sum(s["peer_fills"] for s in stt) > 0
        for s in stt:
            assert s["peer_bytes"] == s["peer_fills"] * PAGE
            assert s["fill_bytes"] + s["peer_bytes"] == s["major"] * PAGE
        assert check_invariants(ap, a, [ra], frames) == []
        assert check_invariants(ap, b, [rb], frames) == []
        ap.ap_region_clear_peers(a, ra)
        ap.ap_region_clear_peers(b, rb)
        ap.ap_munmap(a, ra)
        ap.ap_munmap(b, rb)
    finally:
        teardown(ap, a)
        teardown(ap, b)


def test_peer_argument_errors(ap, dev):
    from paper_conf_isca_shaharbs16_b200._lib import APError
    nbytes = 4 * PAGE
    f = make_file(nbytes, seed=34)
    g = make_file(nbytes + PAGE, seed=34)
    a = ap.ap_cache_create(8, PAGE)
    b = ap.ap_cache_create(8, PAGE)
    c = ap.ap_cache_create(8, 4096)
    peers = [ap.ap_cache_create(2, PAGE) for _ in range(8)]
    try:
        ra, rb, rc = ap.ap_mmap(a, f), ap.ap_mmap(b, f), ap.ap_mmap(c, f)
        rg = ap.ap_mmap(b, g)
        rw = ap.ap_mmap_prot(b, make_file(nbytes, seed=35), ap.AP_PROT_READ | ap.AP_PROT_WRITE)
        for args, code in (((a, ra, a, ra), -1),     # itself
                           ((a, ra, c, rc), -1),     # page size differs
                           ((a, ra, b, rg), -1),     # size differs
                           ((a, ra, b, rw), -1)):    # writable
            with pytest.raises(APError) as e:
                ap.ap_region_add_peer(*args)
            assert e.value.code == code
        rps = [ap.ap_mmap(p, f) for p in peers]
        for p, rp in zip(peers[:7], rps[:7]):
            ap.ap_region_add_peer(a, ra, p, rp)
        with pytest.raises(APError) as e:
            ap.ap_region_add_peer(a, ra, peers[7], rps[7])
        assert e.value.code == -5
        ap.ap_region_clear_peers(a, ra)
        ap.ap_region_add_peer(a, ra, peers[7], rps[7])  # room again
        ap.ap_region_clear_peers(a, ra)
        for p, rp in zip(peers, rps):
            ap.ap_munmap(p, rp)
        for cache, reg in ((a, ra), (b, rb), (c, rc), (b, rg), (b, rw)):
            ap.ap_munmap(cache, reg)
    finally:
        for x in [a, b, c] + peers:
            teardown(ap, x)


def _ipc_exporter(q_handle, q_done, nbytes, npages):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch  # noqa: F401
    import paper_conf_isca_shaharbs16_b200 as ap
    from helpers import make_file
    f = make_file(nbytes, seed=36)
    a = ap.ap_cache_create(npages, PAGE)
    ra = ap.ap_mmap(a, f)
    ap.ap_prefill(a, ra, 0, npages)
    torch.cuda.synchronize()
    q_handle.put(ap.ap_region_export(a, ra))
    q_done.get(timeout=120)  # the importer cleared its peers
    ok = ap.ap_cache_stats(a)["evictions"] == 0
    ap.ap_munmap(a, ra)
    ap.ap_cache_destroy(a)
    q_handle.put(ok)


def test_peer_in_another_process_via_ipc(ap, dev):
    """One process per GPU is how the framework scales: here the peer cache
    lives in a second process on the same GPU and is imported through CUDA
    IPC handles (ap_region_export / ap_region_add_peer_ipc)."""
    npages = 40
    nbytes = npages * PAGE
    ctx = mp.get_context("spawn")
    qh, qd = ctx.Queue(), ctx.Queue()
    p = ctx.Process(target=_ipc_exporter, args=(qh, qd, nbytes, npages))
    p.start()
    try:
        handle = qh.get(timeout=180)
        f = make_file(nbytes, seed=36)
        b = ap.ap_cache_create(16, PAGE)
        try:
            rb = ap.ap_mmap(b, f)
            ap.ap_region_add_peer_ipc(b, rb, handle)
            out = _copy(ap, b, rb, nbytes, dev)
            torch.cuda.synchronize()
            assert ap.ap_last_device_error(b) == 0
            assert np.array_equal(out.cpu().numpy(), f)
            st = ap.ap_cache_stats(b)
            assert st["fill_bytes"] == 0 and st["peer_fills"] == st["major"] >= npages
            assert check_invariants(ap, b, [rb], 16) == []
            ap.ap_region_clear_peers(b, rb)
            ap.ap_munmap(b, rb)
        finally:
            teardown(ap, b)
        qd.put(True)
        assert qh.get(timeout=120) is True
    finally:
        p.join(timeout=60)
        if p.is_alive():
            p.kill()
    assert p.exitcode == 0
