"""Pins for O2 (oracle/invariants.py): a consistent dump passes, and a dump
that breaks each invariant of PAPER.md:113-115/145/157 is rejected."""
import numpy as np

from oracle import invariants as inv


def pte(state, frame=0, rc=0, ref=0):
    return (state << 62) | (ref << 61) | (frame << 32) | rc


def good_dump():
    frames = 4
    ptes = {0: np.array([pte(2, 1), pte(0), pte(2, 3, ref=1)], np.uint64),
            3: np.array([pte(2, 0), pte(0)], np.uint64)}
    owner = np.zeros(frames, np.uint64)
    owner[1] = (1 << 48) | 0
    owner[3] = (1 << 48) | 2
    owner[0] = (4 << 48) | 0
    return ptes, owner, 1, frames


def test_consistent_dump_passes():
    assert inv.check(*good_dump()) == []


def test_fields_roundtrip():
    s, r, f, c = inv.pte_fields(np.array([pte(2, 12345, 77, 1)], np.uint64))
    assert (s[0], r[0], f[0], c[0]) == (2, 1, 12345, 77)


def test_live_refcount_rejected():
    ptes, owner, free_left, frames = good_dump()
    ptes[0][0] = pte(2, 1, rc=3)
    assert any("reference count" in e for e in inv.check(ptes, owner, free_left, frames))
    assert inv.check(ptes, owner, free_left, frames, require_zero_refcounts=False) == []


def test_loading_left_rejected():
    ptes, owner, free_left, frames = good_dump()
    ptes[0][1] = pte(1)
    assert any("LOADING" in e for e in inv.check(ptes, owner, free_left, frames))


def test_double_mapped_frame_rejected():
    ptes, owner, free_left, frames = good_dump()
    ptes[0][1] = pte(2, 3)
    errs = inv.check(ptes, owner, free_left - 1, frames)
    assert any("mapped twice" in e for e in errs)


def test_owner_mismatch_rejected():
    ptes, owner, free_left, frames = good_dump()
    owner[3] = (1 << 48) | 1
    assert any("does not point back" in e for e in inv.check(ptes, owner, free_left, frames))


def test_frame_leak_rejected():
    ptes, owner, free_left, frames = good_dump()
    assert any("conservation" in e for e in inv.check(ptes, owner, 0, frames))


def test_fill_counts():
    assert inv.check_fill_counts({"major": 10, "evictions": 0}, 10, 16, 16) == []
    assert inv.check_fill_counts({"major": 11, "evictions": 0}, 10, 16, 16)
    assert inv.check_fill_counts({"major": 9, "evictions": 0}, 10, 4, 16)
    assert inv.check_fill_counts({"major": 30, "evictions": 20}, 10, 4, 16) == []
