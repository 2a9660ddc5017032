"""Pins for the oracle's O1 (reads) -- checked against things other than the
oracle itself: published generator/checksum vectors, byte-level re-reads of
tiny files through numpy, an inverse enumeration of the SEQ access order,
and closed-form properties of the UNIFORM/DIVERGENT patterns."""
import json
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")
GAMMA = 0x9E3779B97F4A7C15
M64 = (1 << 64) - 1


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def test_splitmix64_published_vectors():
    g = _gold("splitmix64_seed0.json")
    for k, want in enumerate(g["outputs"]):
        assert oracle.sm64((k * GAMMA) & M64) == int(want, 16)
        assert synth.sm64((k * GAMMA) & M64) == int(want, 16)


def test_fnv1a64_published_vectors():
    g = _gold("fnv1a64.json")
    basis = int(g["offset_basis"], 16)
    assert basis == int(g["vectors"][""], 16)
    for msg in ("a", "b"):
        # one-byte message == one zero-extended word (DESIGN.md checksum)
        word = msg.encode() + bytes(7)
        assert oracle.fnv_words(basis, word) == int(g["vectors"][msg], 16)


def test_fnv_four_byte_value_is_zero_extended_word():
    h0 = 0xCBF29CE484222325
    for v in (0, 1, 0xDEADBEEF, 0xFFFFFFFF):
        four = int(v).to_bytes(4, "little")
        assert oracle.fnv_words(h0, four) == oracle.fnv_words(h0, four + bytes(4))


def test_fnv_sixteen_byte_value_is_two_words_low_first():
    h0 = 0xCBF29CE484222325
    lo, hi = 0x0123456789ABCDEF, 0xFEDCBA9876543210
    v = lo.to_bytes(8, "little") + hi.to_bytes(8, "little")
    assert oracle.fnv_words(h0, v) == oracle.fnv_words(oracle.fnv_words(h0, v[:8]), v[8:])
    assert oracle.fnv_words(h0, v) != oracle.fnv_words(oracle.fnv_words(h0, v[8:]), v[:8])


def _py_fnv(values, elem):
    """Independent FNV-1a-64 over words in Python ints (published constants)."""
    h = 0xCBF29CE484222325
    for v in values:
        if elem >= 8:
            words = [int.from_bytes(v[k:k + 8].tobytes(), "little") for k in range(0, elem, 8)]
        else:
            words = [int.from_bytes(v.tobytes(), "little")]
        for w in words:
            h = ((h ^ w) * 0x100000001B3) & M64
    return h


def test_file_generator_words_are_splitmix_counters():
    f = synth.make_file(8 * 10 + 3, seed=77)
    words = f[:80].view(np.uint64)
    for j in range(10):
        assert int(words[j]) == oracle.sm64(77 + j)
    assert f[80:].tobytes() == oracle.sm64(77 + 10).to_bytes(8, "little")[:3]


@pytest.mark.parametrize("elem,unit,span", [(16, 4096, 4 * 4096), (4, 4096, 3 * 4096 + 1000),
                                            (16, 1024, 5 * 1024 + 48)])
def test_seq_copy_is_the_file(elem, unit, span):
    f = synth.make_file(span + 4096, seed=5)
    out = oracle.read_seq(f, span, unit, elem, nthreads=96, passes=1, copy=True)
    # every whole element of [0, span) is read exactly where it lives
    whole = (span // elem) * elem
    assert np.array_equal(out[:whole], f[:whole])
    assert not out[whole:].any()


@pytest.mark.parametrize("elem,unit,nthreads,passes", [(16, 2048, 64, 1), (4, 512, 96, 2),
                                                      (16, 4096, 32, 3)])
def test_seq_checksums_by_inverse_enumeration(elem, unit, nthreads, passes):
    span = 7 * unit + 3 * elem
    f = synth.make_file(span + 64, seed=11)
    ck = oracle.read_seq(f, span, unit, elem, nthreads, passes)
    W = nthreads // 32
    per_thread = {t: [] for t in range(nthreads)}
    # inverse mapping: walk the file element by element and ask who reads it
    for _ in range(passes):
        order = []
        for e in range(span // elem):
            off = e * elem
            u = off // unit
            k = (off % unit) // elem
            t = (u % W) * 32 + k % 32
            order.append((u // W, k // 32, t, off))  # (round, j, thread, off)
        for _, _, t, off in sorted(order):
            per_thread[t].append(f[off:off + elem])
    for t in range(nthreads):
        assert int(ck[t]) == _py_fnv(per_thread[t], elem), t


@pytest.mark.parametrize("elem", [4, 8, 16])
def test_uniform_offsets_and_checksums(elem):
    nbytes = 64 * 1024
    f = synth.make_file(nbytes, seed=3)
    T, R, seed = 64, 5, 1234
    offs = [[oracle.uniform_off(nbytes, elem, seed, t, i) for i in range(R)] for t in range(T)]
    flat = np.array(offs).ravel()
    assert np.all(flat % elem == 0) and np.all(flat + elem <= nbytes)
    assert len(set(flat.tolist())) > 0.9 * flat.size  # draws are spread out
    ck = oracle.read_uniform(f, nbytes, elem, T, R, seed)
    for t in range(T):
        assert int(ck[t]) == _py_fnv([f[o:o + elem] for o in offs[t]], elem)


def test_uniform_offsets_are_uniform():
    nbytes, elem = 4096 * 64, 4
    counts = np.zeros(64, dtype=np.int64)
    for t in range(256):
        for i in range(16):
            counts[oracle.uniform_off(nbytes, elem, 99, t, i) // 4096] += 1
    expected = 256 * 16 / 64
    chi2 = float(((counts - expected) ** 2 / expected).sum())
    assert chi2 < 120  # 63 dof; p ~ 1e-5 threshold


@pytest.mark.parametrize("page,elem", [(4096, 4), (65536, 4), (4096, 16)])
def test_divergent_lanes_on_distinct_pages(page, elem):
    npg = 100
    nbytes = npg * page + 123  # ragged tail is never touched
    for w in range(4):
        for i in range(6):
            offs = [oracle.divergent_off(nbytes, page, elem, 7, w * 32 + l, i) for l in range(32)]
            pages = [o // page for o in offs]
            assert len(set(pages)) == 32
            assert all(o % elem == 0 and o + elem <= npg * page for o in offs)


def test_divergent_checksums():
    page, elem, npg = 4096, 4, 40
    nbytes = npg * page
    f = synth.make_file(nbytes, seed=8)
    ck = oracle.read_divergent(f, nbytes, page, elem, 64, 3, 42)
    for t in range(64):
        offs = [oracle.divergent_off(nbytes, page, elem, 42, t, i) for i in range(3)]
        assert int(ck[t]) == _py_fnv([f[o:o + elem] for o in offs], elem)
