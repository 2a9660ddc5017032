"""Randomised stress of the whole fault path (seeded, reproducible): random
file sizes (ragged), page sizes, cache sizes down to one frame, launch
shapes, patterns, element sizes, eviction policies, and interleaved writes.
Every configuration must match the oracle bit for bit and leave the page
cache consistent (O1, O1', O2)."""
import numpy as np
import pytest
import torch

import oracle
from helpers import check_invariants, make_file, teardown

pytestmark = pytest.mark.gpu

# AP_STRESS_CASES="a-b" (a soak run): seeds a .. b-1 instead of the 24 default
_rng = __import__("os").environ.get("AP_STRESS_CASES")
CASES = list(range(*map(int, _rng.split("-")))) if _rng else list(range(24))


def _cfg(seed):
    rng = np.random.default_rng(1000 + seed)
    page = int(rng.choice([4096, 16384, 65536]))
    npg = int(rng.integers(40, 200))
    nbytes = npg * page - int(rng.integers(0, page // 16)) * 16
    frames = int(rng.choice([1, 2, 5, 17, 64, 1024]))
    block = int(rng.choice([32, 64, 128, 256, 512]))
    grid = int(rng.integers(1, 12))
    elem = int(rng.choice([4, 8, 16]))
    policy = int(rng.integers(0, 2))
    return rng, page, nbytes, frames, block, grid, elem, policy


@pytest.mark.parametrize("case", CASES)
def test_random_config(ap, case):
    rng, page, nbytes, frames, block, grid, elem, policy = _cfg(case)
    f = make_file(nbytes, seed=case)
    writable = case % 3 == 0
    cache = ap.ap_cache_create(frames, page)
    try:
        ap.ap_cache_set_policy(cache, policy, case)
        ap.ap_cache_set_tuning(cache, int(rng.integers(1, 4)), 64, 0)
        r = ap.ap_mmap_prot(cache, f, 3 if writable else 1)
        cur = f.copy()
        nthreads = grid * block
        dev = torch.device("cuda:0")
        for step in range(3):
            kind = int(rng.integers(0, 4 if writable else 3))
            seed = int(rng.integers(0, 1 << 30))
            if kind == 0:  # UNIFORM reads
                reads = int(rng.integers(1, 6))
                out = torch.zeros(nthreads, dtype=torch.int64, device=dev)
                ap.ap_bench_read(cache, r, ap.bench_cfg(ap.AP_UNIFORM, elem, grid, block,
                                                        reads_per_thread=reads, seed=seed), out)
                torch.cuda.synchronize()
                assert np.array_equal(out.cpu().numpy().view(np.uint64),
                                      oracle.read_uniform(cur, nbytes, elem, nthreads, reads, seed))
            elif kind == 1:  # DIVERGENT reads
                reads = int(rng.integers(1, 4))
                out = torch.zeros(nthreads, dtype=torch.int64, device=dev)
                ap.ap_bench_read(cache, r, ap.bench_cfg(ap.AP_DIVERGENT, elem, grid, block,
                                                        reads_per_thread=reads, page_bytes=page,
                                                        seed=seed), out)
                torch.cuda.synchronize()
                assert np.array_equal(out.cpu().numpy().view(np.uint64),
                                      oracle.read_divergent(cur, nbytes, page, elem, nthreads,
                                                            reads, seed))
            elif kind == 2:  # SEQ reads, random access style
                unit = int(rng.choice([u for u in (512 * elem // 4, 1024, 4096, page)
                                       if u % (32 * elem) == 0 and page % u == 0]))
                acc = int(rng.integers(0, 3))
                out = torch.zeros(nthreads, dtype=torch.int64, device=dev)
                ap.ap_bench_read(cache, r, ap.bench_cfg(ap.AP_SEQ, elem, grid, block,
                                                        unit_bytes=unit, access=acc), out)
                torch.cuda.synchronize()
                assert np.array_equal(out.cpu().numpy().view(np.uint64),
                                      oracle.read_seq(cur, nbytes, unit, elem, nthreads, 1))
            else:  # scattered writes
                reads = int(rng.integers(1, 4))
                if nthreads * reads <= nbytes // elem:
                    ap.ap_bench_write(cache, r, ap.bench_cfg(ap.AP_UNIFORM, elem, grid, block,
                                                             reads_per_thread=reads, seed=seed))
                    torch.cuda.synchronize()
                    cur = oracle.apply_writes(cur, elem, 1, nthreads=nthreads, reads=reads,
                                              seed=seed)
            assert ap.ap_last_device_error(cache) == 0
            assert check_invariants(ap, cache, [r], frames) == []
        ap.ap_munmap(cache, r)
        if writable:
            assert np.array_equal(f, cur)
    finally:
        teardown(ap, cache)
