"""Pins for the oracle's O3 (collage) -- against the
hand-worked fixture in tests/golden/, closed forms, a numpy per-pixel recount,
Python's floor division, and numpy brute-force nearest neighbour in the
degenerate one-bucket LSH (which turns the collage into textbook exhaustive
search)."""
import json
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _hist_numpy(img, b):
    """Independent recount: np.bincount over the block's pixels per channel."""
    H, W, _ = img.shape
    bw = W // 32
    by, bx = divmod(b, bw)
    blk = img[by * 32:(by + 1) * 32, bx * 32:(bx + 1) * 32, :]
    return np.concatenate([np.bincount(blk[:, :, c].ravel(), minlength=256) for c in range(3)])


def test_hist_golden_fixture():
    g = json.load(open(os.path.join(GOLD, "collage_hist_2blocks.json")))
    img = np.zeros((32, 64, 3), dtype=np.uint8)
    img[:, :32] = (10, 20, 30)
    img[:, 48:] = (255, 128, 7)
    for b, key in ((0, "block0"), (1, "block1")):
        h = oracle.block_hist(img, b)
        want = np.zeros(768, dtype=np.int64)
        for k, v in g["expected_nonzero_bins"][key].items():
            want[int(k)] = v
        assert np.array_equal(h.astype(np.int64), want)
    h0, h1 = oracle.block_hist(img, 0), oracle.block_hist(img, 1)
    assert oracle.ssd(h0, h1) == int(g["ssd_block0_block1"].split("=")[-1])


def test_hist_channel_sums_and_recount():
    img = np.random.default_rng(0).integers(0, 256, size=(96, 128, 3), dtype=np.uint8)
    for b in range(12):
        h = oracle.block_hist(img, b)
        assert [int(h[c * 256:(c + 1) * 256].sum()) for c in range(3)] == [1024] * 3
        assert np.array_equal(h.astype(np.int64), _hist_numpy(img, b))


def test_ssd_closed_forms():
    rng = np.random.default_rng(1)
    a = rng.integers(0, 1025, 768).astype(np.uint32)
    b = rng.integers(0, 1025, 768).astype(np.uint32)
    assert oracle.ssd(a, a) == 0
    assert oracle.ssd(a, b) == oracle.ssd(b, a)
    for d, delta in ((0, 1), (255, 7), (767, 1000)):
        c = a.copy()
        c[d] = a[d] + delta
        assert oracle.ssd(a, c) == delta * delta
    lo = np.zeros(768, np.uint32); hi = np.zeros(768, np.uint32)
    lo[[0, 256, 512]] = 1024
    hi[[1, 257, 513]] = 1024
    assert oracle.ssd(lo, hi) == 6 * 1024 ** 2  # the uint32 maximum of R-A2


def test_floordiv_matches_python():
    rng = np.random.default_rng(2)
    for a in list(rng.integers(-10**7, 10**7, 500)) + [-1, 0, 1, -7, 7, -14, 14]:
        for w in (1, 3, 7, 1000, 4096):
            assert oracle.floordiv(int(a), w) == int(a) // w


def test_lsh_key_k0_is_constant_bucket():
    rng = np.random.default_rng(3)
    proj = np.zeros((3, 0, 768), np.int16); bias = np.zeros((3, 0), np.int32)
    for t in range(3):
        want = oracle.sm64(t) >> (64 - 12)
        for _ in range(4):
            h = rng.integers(0, 50, 768).astype(np.uint32)
            assert oracle.lsh_key(h, t, proj, bias, 100, 12) == want


@pytest.mark.parametrize("sign", [1, -1])
def test_lsh_key_unit_projection(sign):
    """proj[t][k] = sign * e_d  =>  h_k = floor((sign*hist[d] + bias)/w)."""
    L, K, w, bb = 2, 3, 50, 16
    proj = np.zeros((L, K, 768), np.int16)
    bias = np.zeros((L, K), np.int32)
    dims = [[5, 300, 700], [1, 2, 767]]
    for t in range(L):
        for k in range(K):
            proj[t, k, dims[t][k]] = sign
            bias[t, k] = 7 * (t + 1) + k
    rng = np.random.default_rng(4)
    for _ in range(10):
        h = rng.integers(0, 1025, 768).astype(np.uint32)
        for t in range(L):
            x = oracle.sm64(t)
            for k in range(K):
                hk = (sign * int(h[dims[t][k]]) + int(bias[t, k])) // w
                x = oracle.sm64(x ^ (hk & 0xFFFFFFFF))
            assert oracle.lsh_key(h, t, proj, bias, w, bb) == x >> (64 - bb)
            # bins the projection does not look at cannot change the key
            h2 = h.copy()
            other = [d for d in range(768) if d not in dims[t]][:50]
            h2[other] = rng.integers(0, 1025, len(other))
            assert oracle.lsh_key(h2, t, proj, bias, w, bb) == oracle.lsh_key(h, t, proj, bias,
                                                                               w, bb)


def test_lsh_key_depends_on_table_and_projection_order():
    proj, bias = synth.make_lsh_params(2, 4, 500, seed=9)
    h = oracle.block_hist(np.random.default_rng(5).integers(0, 256, (32, 32, 3), np.uint8), 0)
    k0 = oracle.lsh_key(h, 0, proj, bias, 500, 20)
    k1 = oracle.lsh_key(h, 1, proj, bias, 500, 20)
    assert k0 != k1
    swapped = proj[:, ::-1, :].copy()
    assert oracle.lsh_key(h, 0, swapped, bias[:, ::-1].copy(), 500, 20) != k0


def _dataset(n, seed=21, stride=4096):
    f = synth.make_records(n, stride, seed)
    recs = np.stack([f[i * stride:i * stride + 3072].view(np.uint32) for i in range(n)])
    return f, recs


def test_records_are_colour_counts_with_zero_padding():
    f, recs = _dataset(64)
    assert np.all(recs.reshape(64, 3, 256).sum(axis=2) == 1024)
    pad = f.reshape(64, 4096)[:, 3072:]
    assert not pad.any()


def test_build_index_is_a_partition_by_key():
    n, bb = 2000, 8
    f, recs = _dataset(n)
    proj, bias = synth.make_lsh_params(3, 4, 2000, seed=10)
    off, ids = oracle.build_index(f, 4096, n, proj, bias, 2000, bb)
    B = 1 << bb
    for t in range(3):
        assert off[t, 0] == 0 and off[t, B] == n and np.all(np.diff(off[t].astype(np.int64)) >= 0)
        assert np.array_equal(np.sort(ids[t]), np.arange(n))
        for key in range(B):
            seg = ids[t, off[t, key]:off[t, key + 1]]
            assert np.all(np.diff(seg.astype(np.int64)) > 0)  # ascending ids
            for i in seg[:3]:
                assert oracle.lsh_key(recs[i], t, proj, bias, 2000, bb) == key


def _bruteforce(img, recs):
    """Exhaustive nearest neighbour with numpy: (SSD, index) lexicographic."""
    H, W, _ = img.shape
    nb = (W // 32) * (H // 32)
    out = np.empty((nb, 2), np.int64)
    r = recs.astype(np.int64)
    for b in range(nb):
        q = _hist_numpy(img, b).astype(np.int64)
        d = ((r - q) ** 2).sum(axis=1)
        i = int(np.lexsort((np.arange(len(d)), d))[0])
        out[b] = (i, d[i])
    return out


def test_degenerate_lsh_is_exhaustive_search():
    n = 4096
    f, recs = _dataset(n)
    img, src, is_copy = synth.make_target(256, 256, n, ds_seed=21, seed=3, pool=16,
                                          copy_permille=200)
    proj = np.zeros((1, 0, 768), np.int16); bias = np.zeros((1, 0), np.int32)
    off, ids = oracle.build_index(f, 4096, n, proj, bias, 1, 4)
    win = oracle.collage(img, proj, bias, 1, 4, f, 4096, n, off, ids)
    assert np.array_equal(win.astype(np.int64), _bruteforce(img, recs))


def test_planted_copies_find_themselves():
    n = 3000
    f, recs = _dataset(n, seed=33)
    proj, bias = synth.make_lsh_params(4, 8, 3000, seed=1)
    off, ids = oracle.build_index(f, 4096, n, proj, bias, 3000, 10)
    img, src, is_copy = synth.make_target(512, 256, n, ds_seed=33, seed=8, pool=32,
                                          copy_permille=300)
    win = oracle.collage(img, proj, bias, 3000, 10, f, 4096, n, off, ids)
    assert is_copy.sum() > 10
    for b in np.nonzero(is_copy)[0]:
        same = np.nonzero(np.all(recs == recs[src[b]], axis=1))[0]
        assert tuple(win[b]) == (int(same.min()), 0)


def test_winner_is_lexicographic_min_over_candidates():
    n, bb, w = 3000, 9, 1500
    f, recs = _dataset(n, seed=44)
    proj, bias = synth.make_lsh_params(3, 6, w, seed=2)
    off, ids = oracle.build_index(f, 4096, n, proj, bias, w, bb)
    img, _, _ = synth.make_target(256, 128, n, ds_seed=44, seed=9, pool=8, copy_permille=0)
    win = oracle.collage(img, proj, bias, w, bb, f, 4096, n, off, ids)
    for b in range(win.shape[0]):
        q = _hist_numpy(img, b).astype(np.int64)
        cands = set()
        for t in range(3):
            key = oracle.lsh_key(q.astype(np.uint32), t, proj, bias, w, bb)
            cands.update(ids[t, off[t, key]:off[t, key + 1]].tolist())
        if not cands:
            assert tuple(win[b]) == (oracle.EMPTY, oracle.EMPTY)
            continue
        best = min((int(((recs[i].astype(np.int64) - q) ** 2).sum()), i) for i in cands)
        assert (int(win[b, 1]), int(win[b, 0])) == best
