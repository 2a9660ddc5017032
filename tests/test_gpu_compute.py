"""Fig. 6 workloads (NEXT N4): the apointer version equals
its raw twin bit for bit and both equal the oracle (FFT within float error)."""
import numpy as np
import pytest
import torch

import oracle
from helpers import make_file, teardown

pytestmark = pytest.mark.gpu

WORKS = ["add", "read", "random", "reduce", "fft", "bitonic"]


@pytest.mark.parametrize("work", WORKS)
@pytest.mark.parametrize("elem", [4, 16])
def test_workload_parity(ap, work, elem):
    page = 65536
    span = 32 * page
    f = make_file(2 * span, seed=3)
    cache = ap.ap_cache_create(16, page)  # half the pages fit: faults + evictions
    try:
        r = ap.ap_mmap(cache, f)
        grid, block = 3, 256
        n = grid * block
        out = torch.zeros(n, dtype=torch.int64, device="cuda")
        ap.ap_bench_compute(cache, r, work, elem, grid, block, span, out, iters=7)
        dcopy = torch.from_numpy(f).to("cuda")
        raw = torch.zeros_like(out)
        ap.ap_bench_compute(cache, r, work, elem, grid, block, span, raw, iters=7,
                            mode=ap.AP_MODE_RAW, raw_base=dcopy)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0
        assert torch.equal(out, raw)
        got = out.cpu().numpy().view(np.uint64).astype(np.float64)
        want = oracle.compute(f, span, page, elem, n, ap.WORKS[work], iters=7)
        if work == "fft":
            assert np.allclose(got, want, rtol=1e-4, atol=64 * span / page)
        elif work in ("read", "add", "bitonic", "reduce", "random"):
            # exact modulo 2^64 (accumulators are uint64; oracle sums are < 2^53)
            assert np.array_equal(got, want)
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)
