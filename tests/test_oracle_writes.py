"""Pins for the writes oracle (apply_writes): coverage, bijectivity of the
race-free permutation, and values from the published splitmix64 vectors."""
import numpy as np

import oracle
import synth

GAMMA = 0x9E3779B97F4A7C15


def test_perm_is_a_bijection():
    for M in (7, 64, 1000, 4096, 1 << 16):
        got = sorted(oracle.perm_idx(k, M) for k in range(M))
        assert got == list(range(M))


def test_seq_writes_cover_exactly_the_span():
    f = synth.make_file(4096 + 40, seed=2)
    out = oracle.apply_writes(f, 16, 0, span=4096 + 40, seed=5)
    assert np.all(out[4096 + 32:] == f[4096 + 32:])  # the ragged 8 bytes are untouched
    changed = (out[:4096 + 32].reshape(-1, 16) != f[:4096 + 32].reshape(-1, 16)).any(axis=1)
    assert changed.mean() > 0.99


def test_written_values_follow_splitmix():
    f = np.zeros(64, np.uint8)
    out = oracle.apply_writes(f, 4, 0, span=64, seed=0)
    # element e holds the low 32 bits of sm64(0 ^ e); e = 0 -> published output 0
    assert int(out[:4].view(np.uint32)[0]) == 0xE220A8397B1DCDAF & 0xFFFFFFFF
    out8 = oracle.apply_writes(np.zeros(16, np.uint8), 8, 0, span=16, seed=GAMMA)
    # sm64(GAMMA ^ 0) = published output 1, sm64(GAMMA ^ 1) is its neighbour
    assert int(out8[:8].view(np.uint64)[0]) == 0x6E789E6AA1B965F4


def test_uniform_writes_touch_distinct_elements():
    f = np.zeros(4096, np.uint8)
    out = oracle.apply_writes(f, 4, 1, nthreads=64, reads=16, seed=9)
    assert int((out.view(np.uint32) != 0).sum()) == 64 * 16
