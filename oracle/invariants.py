"""O2 -- fault-path invariants, checked on a dump of the page cache taken
after a kernel has finished (TEST INFRASTRUCTURE ONLY, see oracle/__init__.py).

These are not values the method computes but the properties the paper fixes
for its page cache:

* a page with a positive reference count cannot be evicted, and the count is
  the number of linked apointers on the page (§III-B/C),
  so once every apointer is destroyed every count is zero;
* a warp's faults are handled by a single leader per page, incrementing the
  count once by the number of lanes on the page (§III-D), so a
  page is brought in once per major fault and the cache never holds a page
  twice;
* frame bookkeeping (R-A17/A18 in DESIGN.md): a frame is either still on the
  free list or owned by exactly one VALID PTE, and the owner table points back.

Dump format (the C-ABI's ap_cache_dump / ap_region_dump_pte, include/ap.h):
  pte[r]   uint64[npages_r]   bits 63:62 state (0 EMPTY, 1 LOADING, 2 VALID),
                              bit 61 reference bit, bit 60 dirty, bits 59:32 frame,
                              bits 31:0 reference count
  owner    uint64[frames]     0 = none, else ((region+1) << 48) | page
  free_left int               frames still on the free list
"""
import numpy as np

EMPTY, LOADING, VALID = 0, 1, 2


def pte_fields(pte):
    pte = np.asarray(pte, dtype=np.uint64)
    state = (pte >> np.uint64(62)).astype(np.int64)
    ref = ((pte >> np.uint64(61)) & np.uint64(1)).astype(np.int64)
    frame = ((pte >> np.uint64(32)) & np.uint64((1 << 28) - 1)).astype(np.int64)
    rc = (pte & np.uint64(0xFFFFFFFF)).astype(np.int64)
    return state, ref, frame, rc


def check(ptes, owner, free_left, frames, require_zero_refcounts=True):
    """Return a list of violated invariants (empty list == all hold).

    ptes: dict region_id -> uint64 PTE array; owner: uint64[frames]."""
    errs = []
    owner = np.asarray(owner, dtype=np.uint64)
    if owner.shape != (frames,):
        return [f"owner table has shape {owner.shape}, expected ({frames},)"]
    seen_frames = {}
    n_valid = 0
    for r, pte in ptes.items():
        state, ref, frame, rc = pte_fields(pte)
        if np.any(state == 3):
            errs.append(f"region {r}: PTE with undefined state 3")
        if np.any(state == LOADING):
            errs.append(f"region {r}: {int(np.sum(state == LOADING))} PTE(s) left LOADING")
        if require_zero_refcounts and np.any(rc != 0):
            errs.append(f"region {r}: live reference count sum {int(rc.sum())} != 0 "
                        f"(PAPER.md:145: counts drop when apointers are destroyed)")
        empty = state == EMPTY
        if np.any(rc[empty] != 0):
            errs.append(f"region {r}: EMPTY PTE with nonzero reference count")
        vidx = np.nonzero(state == VALID)[0]
        n_valid += len(vidx)
        for pg in vidx:
            f = int(frame[pg])
            if f >= frames:
                errs.append(f"region {r} page {pg}: frame {f} out of range")
                continue
            if f in seen_frames:
                errs.append(f"frame {f} mapped twice: {seen_frames[f]} and {(r, int(pg))}")
            seen_frames[f] = (r, int(pg))
            want = ((r + 1) << 48) | int(pg)
            if int(owner[f]) != want:
                errs.append(f"frame {f}: owner {int(owner[f]):#x} does not point back to "
                            f"region {r} page {pg}")
    if free_left + n_valid != frames:
        errs.append(f"frame conservation: {free_left} free + {n_valid} VALID != {frames} frames")
    return errs


def link_events(offsets, log2_page, warp=32):
    """Closed-form number of page links a per-access run performs
    (Listing 1): `offsets` is
    uint64[nthreads, reads], the offset each thread reads in access order,
    threads numbered so that warp w holds threads 32w .. 32w+31.  A thread
    whose read i lies on the page its read i-1 was on stays linked (no event,
    PAPER.md:147); every other read needs a link, and at iteration i each
    distinct page among a warp's needing lanes is linked once, by one leader
    for the whole group (the count grows by the group size in one step,
    PAPER.md:157).  So events = sum over (warp, i) of the number of distinct
    pages among the warp's lanes that left their page (or start, i = 0).
    With a cache that never runs out of frames each event is exactly one
    major or one minor fault."""
    pg = np.asarray(offsets, dtype=np.uint64) >> np.uint64(log2_page)
    n, reads = pg.shape
    assert n % warp == 0, "whole warps only"
    need = np.ones_like(pg, dtype=bool)
    need[:, 1:] = pg[:, 1:] != pg[:, :-1]
    key = np.where(need, pg.astype(np.int64), -1)
    key = key.reshape(n // warp, warp, reads).transpose(0, 2, 1)   # [warp, i, lane]
    key = np.sort(key, axis=2)
    distinct = (key[:, :, 1:] != key[:, :, :-1]) & (key[:, :, 1:] >= 0)
    return int(distinct.sum() + (key[:, :, 0] >= 0).sum())


def check_link_count(stats_before, stats_after, expected):
    """With enough frames (no frame pressure, no eviction) every page link of
    the run is exactly one major or one minor fault."""
    got = (stats_after["major"] - stats_before["major"]) + \
          (stats_after["minor"] - stats_before["minor"])
    if got != expected:
        return [f"major+minor = {got} link events, closed form {expected}"]
    return []


def check_fill_counts(stats, distinct_pages, frames, npages_total):
    """Fills happen at least once per distinct page touched, and exactly once
    when the cache can hold every page (no eviction): the LOADING claim
    dedupes concurrent faulters of one page (R-A12)."""
    errs = []
    if stats["major"] < distinct_pages:
        errs.append(f"{stats['major']} fills < {distinct_pages} distinct pages touched")
    if frames >= npages_total and stats["major"] != distinct_pages:
        errs.append(f"cache holds every page but {stats['major']} fills != "
                    f"{distinct_pages} distinct pages")
    if frames >= npages_total and stats["evictions"] != 0:
        errs.append(f"{stats['evictions']} evictions although the cache holds every page")
    return errs
