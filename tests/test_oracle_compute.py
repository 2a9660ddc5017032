"""Pins for the compute-workload oracle (Fig. 6 workloads)."""
import numpy as np

import oracle

P = 4096


def _file(words):
    return np.ascontiguousarray(np.asarray(words, dtype=np.uint32)).view(np.uint8)


def test_read_and_add_sum_the_lanes_words():
    w = np.arange(2 * P // 4, dtype=np.uint32)
    f = _file(w)
    acc = oracle.compute(f, P, P, 4, 32, 1)
    # lane l reads words l, l+32, ... of the first page
    want = [float(w[:P // 4][l::32].sum()) for l in range(32)]
    assert np.array_equal(acc, want)
    acc2 = oracle.compute(f, P, P, 4, 32, 0)
    want2 = [float(w[:P // 4][l::32].sum() + w[P // 4:][l::32].sum()) for l in range(32)]
    assert np.array_equal(acc2, want2)


def test_random_lcg_first_step():
    # Numerical Recipes LCG: x1 = 1664525*x0 + 1013904223 (mod 2^32); from 0 -> 1013904223
    f = _file(np.zeros(P // 4, np.uint32))
    acc = oracle.compute(f, P, P, 4, 32, 2, iters=1)
    assert np.all(acc == 1013904223.0 * (P // 4 // 32))


def test_reduce_gives_every_lane_the_warp_sum():
    w = np.random.default_rng(1).integers(0, 1000, P // 4).astype(np.uint32)
    acc = oracle.compute(_file(w), P, P, 4, 32, 3)
    assert np.all(acc == float(w.sum()))


def test_fft_of_constant_is_an_impulse():
    # x[n] = 3 + 0i  ->  X[0] = 96, X[k>0] = 0;  power/65536 floored
    f = _file(np.full(P // 4, 3, np.uint32))
    acc = oracle.compute(f, P, P, 4, 32, 4)
    reps = P // 4 // 32
    assert acc[0] == reps * np.floor(96.0 ** 2 / 65536.0) == 0
    f = _file(np.full(P // 4, 1000, np.uint32))
    acc = oracle.compute(f, P, P, 4, 32, 4)
    assert acc[0] == reps * np.floor(32000.0 ** 2 / 65536.0)
    assert np.all(acc[1:] == 0)


def test_bitonic_weights_sorted_values():
    w = np.tile(np.arange(31, -1, -1, dtype=np.uint32), P // 4 // 32)
    acc = oracle.compute(_file(w), P, P, 4, 32, 5)
    reps = P // 4 // 32
    assert np.array_equal(acc, [reps * l * (l + 1) for l in range(32)])
