"""Pins for O2 (oracle/invariants.py): a consistent dump passes, and a dump
that breaks each invariant of PAPER.md:113-115/145/157 is rejected."""
import numpy as np
import pytest

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


def _link_events_brute(offs, lg):
    """Listing 1 walked by hand: per warp and iteration,
    the set of pages whose lanes are not linked to them yet."""
    n, reads = offs.shape
    events = 0
    linked = [None] * n
    for w in range(n // 32):
        for i in range(reads):
            need = set()
            for lane in range(32):
                t = 32 * w + lane
                p = int(offs[t, i]) >> lg
                if linked[t] != p:
                    need.add(p)
                    linked[t] = p
            events += len(need)
    return events


def test_link_events_closed_forms():
    """one leader (one link) per distinct page per warp."""
    from oracle.invariants import link_events
    lg = 12
    reads, warps = 5, 3
    n = 32 * warps
    # every lane of a warp on the same page, a new page each iteration
    same = np.array([[((w * 100 + i) << lg) + 4 * (t % 32) for i in range(reads)]
                     for t in range(n) for w in [t // 32]], dtype=np.uint64)
    assert link_events(same, lg) == warps * reads
    # 32 distinct pages per warp-iteration
    dist = np.array([[((t * 1000 + i) << lg) for i in range(reads)] for t in range(n)],
                    dtype=np.uint64)
    assert link_events(dist, lg) == 32 * warps * reads
    # lanes that stay on their page never link again
    stay = np.array([[(t << lg) + 8 * i for i in range(reads)] for t in range(n)],
                    dtype=np.uint64)
    assert link_events(stay, lg) == 32 * warps
    # leaving a page and coming back is a new link (the pointer was unlinked)
    back = np.array([[((i % 2) << lg) for i in range(reads)] for t in range(32)],
                    dtype=np.uint64)
    assert link_events(back, lg) == reads


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_link_events_brute_force(seed):
    from oracle.invariants import link_events
    rng = np.random.default_rng(seed)
    offs = rng.integers(0, 1 << 18, size=(64, 7), dtype=np.uint64)  # 64 pages of 4 KiB
    assert link_events(offs, 12) == _link_events_brute(offs, 12)


def test_offsets_match_the_per_read_generator():
    import oracle
    for pattern, page in ((1, 0), (2, 4096)):
        offs = oracle.offsets(pattern, 1 << 22, 4, 64, 3, 5, page)
        for t in (0, 31, 63):
            for i in range(3):
                want = (oracle.uniform_off(1 << 22, 4, 5, t, i) if pattern == 1 else
                        oracle.divergent_off(1 << 22, page, 4, 5, t, i))
                assert int(offs[t, i]) == want
