"""Randomised stress of the collage path (seeded, reproducible; PAPER.md:
409-419): random dataset sizes, record strides (aligned 4 KiB or straddling
pages), page and cache sizes, LSH shapes, candidate groupings, schedules,
record-id windows (fused launches, precomputed window bounds, empty-window
exits) and unit / record-id partitions folded with AP_COLLAGE_ACCUMULATE.
Winners must equal the oracle's, computed on the oracle's own bucket index,
bit for bit, and the page cache must stay consistent (O2).
AP_STRESS_CASES="a-b" runs seeds a .. b-1 (a soak run) instead of the 12
default ones."""
import os

import numpy as np
import pytest
import torch

import oracle
import synth
from helpers import check_invariants, make_records, teardown
from paper_conf_isca_shaharbs16_b200 import mgpu

pytestmark = pytest.mark.gpu

_rng = os.environ.get("AP_STRESS_CASES")
CASES = list(range(*map(int, _rng.split("-")))) if _rng else list(range(12))


def _cfg(seed):
    rng = np.random.default_rng(5000 + seed)
    n = int(rng.integers(300, 4000))
    stride = int(rng.choice([4096, 3072, 3584, 5120]))
    page = int(rng.choice([4096, 8192, 65536]))
    L = int(rng.integers(1, 5))
    K = int(rng.integers(0, 6))
    bb = int(rng.integers(3, 11))
    W = 32 * int(rng.integers(1, 9))
    H = 32 * int(rng.integers(1, 9))
    group = int(rng.choice([1, 2, 4, 8, 16, 32]))
    schedule = int(rng.integers(0, 4))
    chunks = int(rng.choice([0, 0, 2, 5, 17, 64])) if schedule in (2, 3) else 0
    file_pages = (n * stride + page - 1) // page
    frames = int(rng.choice([3, 8, 40, max(3, file_pages // 3), file_pages + 8]))
    parts = int(rng.choice([1, 1, 2, 3])) if schedule in (2, 3) else 1
    return dict(n=n, stride=stride, page=page, L=L, K=K, bb=bb, W=W, H=H, group=group,
                schedule=schedule, chunks=chunks, frames=frames, parts=parts,
                seed=int(rng.integers(1, 1 << 30)))


@pytest.mark.parametrize("case", CASES)
def test_random_collage(ap, case):
    c = _cfg(case)
    dev = torch.device("cuda:0")
    n, stride, w = c["n"], c["stride"], 2500
    recs = make_records(n, stride, c["seed"])
    proj, bias = synth.make_lsh_params(c["L"], c["K"], w, seed=c["seed"] + 1)
    img, _, _ = synth.make_target(c["W"], c["H"], n, ds_seed=c["seed"], seed=c["seed"] + 2,
                                  pool=16, copy_permille=100)
    cache = ap.ap_cache_create(c["frames"], c["page"])
    try:
        r = ap.ap_mmap(cache, recs)
        bb, L, K = c["bb"], c["L"], c["K"]
        off = torch.zeros((L, (1 << bb) + 1), dtype=torch.int32, device=dev)
        ids = torch.zeros((L, n), dtype=torch.int32, device=dev)
        pd = torch.from_numpy(proj).to(dev)
        bd = torch.from_numpy(bias).to(dev)
        ap.ap_lsh_build_index(cache, r, n, stride, L, K, bb, w, pd, bd, off, ids)
        tgt = torch.from_numpy(img).to(dev)
        nb = (c["W"] // 32) * (c["H"] // 32)
        win = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        if c["parts"] == 1:
            ap.ap_collage_run(cache, r, ap.collage_in(tgt, c["W"], c["H"], pd, bd, w, bb, off, ids,
                                                      n, stride, group=c["group"],
                                                      schedule=c["schedule"],
                                                      id_chunks=c["chunks"]), win)
        else:
            # record-id slices folded into one array (the multi-GPU combine)
            ap.ap_winners_init(win, nb)
            for g in range(c["parts"]):
                i0, i1 = mgpu.id_range(n, g, c["parts"])
                if i1 <= i0:
                    continue
                ap.ap_collage_run(cache, r, ap.collage_in(
                    tgt, c["W"], c["H"], pd, bd, w, bb, off, ids, n, stride, group=c["group"],
                    schedule=c["schedule"], id_chunks=min(c["chunks"], i1 - i0),
                    id_begin=i0, id_end=i1, flags=ap.AP_COLLAGE_ACCUMULATE), win)
        torch.cuda.synchronize()
        assert ap.ap_last_device_error(cache) == 0, c
        o_off, o_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
        want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, o_off, o_ids)
        assert np.array_equal(win.cpu().numpy().view(np.uint32), want), c
        assert check_invariants(ap, cache, [r], c["frames"]) == [], c
        ap.ap_munmap(cache, r)
    finally:
        teardown(ap, cache)
