"""CPU oracle for the apointer dereference path and the photo collage.

TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / `--impl reference` legs may import this package. The product
path (paper_conf_isca_shaharbs16_b200) never imports it, and it shares no code
with the CUDA sources.

What it computes (citations are PAPER.md lines; readings R-Ax are DESIGN.md's):

* O1 reads -- plain file indexing (PAPER.md:121 apointers "behave just like
  regular memory pointers"; PAPER.md:141-143 faults are invisible to values).
  Pinned by tests/test_oracle_reads.py: the splitmix64 and FNV-1a-64 published
  test vectors, brute-force re-reads through numpy views on tiny files, and
  closed-form access-pattern properties (distinct pages per warp, coverage).
* O1' writes -- the file with each stored element replaced (plain
  indexing; Fig. 3 `*ptr = 25`).  Pinned by the published
  splitmix vectors, coverage of the SEQ pattern and bijectivity of the
  permutation pattern (tests/test_oracle_writes.py).
* compute workloads (Fig. 6) -- Add/Read/Random-N/Reduce/
  FFT/Bitonic accumulators from their definitions (FFT as the O(n^2) DFT in
  float64).  Pinned by closed forms in tests/test_oracle_compute.py (a
  constant vector's DFT is an impulse, sorted input is a fixed point of the
  sort, the LCG's published first step).
* O2 fault-path invariants -- `invariants.py`.
  Pinned by negative tests: a dump that breaks each invariant is rejected.
* O3 collage -- histogram -> LSH keys -> candidate buckets
  -> squared Euclidean distance -> lexicographic argmin. Pinned by
  tests/test_oracle_collage.py: channel sums = 1024, a per-pixel recount, SSD
  closed forms, floor division against Python's //, the degenerate LSH (one
  bucket) == numpy brute-force nearest neighbour, planted self-queries, and
  the hand-worked fixtures under tests/golden/.

Parity pins cover every function exported here; none is "parity unpinned".
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

EMPTY = 0xFFFFFFFF


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `make` (or __graft_entry__.build())")
        lib = ctypes.CDLL(_LIB_PATH)
        u64, u32, i32, i64, vp, ci = (ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int32,
                                      ctypes.c_int64, ctypes.c_void_p, ctypes.c_int)
        lib.or_sm64.restype = u64
        lib.or_sm64.argtypes = [u64]
        lib.or_fnv_words.restype = u64
        lib.or_fnv_words.argtypes = [u64, vp, u32]
        lib.or_read_seq.argtypes = [vp, u64, u32, u32, u64, u32, vp, vp, ci]
        lib.or_uniform_off.restype = u64
        lib.or_uniform_off.argtypes = [u64, u32, u64, u64, u64]
        lib.or_read_uniform.argtypes = [vp, u64, u32, u64, u32, u64, vp, ci]
        lib.or_divergent_off.restype = u64
        lib.or_divergent_off.argtypes = [u64, u32, u32, u64, u64, u64]
        lib.or_read_divergent.argtypes = [vp, u64, u32, u32, u64, u32, u64, vp, ci]
        lib.or_offsets.argtypes = [ci, u64, u32, u32, u64, u64, u32, vp]
        lib.or_block_hist.argtypes = [vp, u32, u32, u64, vp]
        lib.or_floordiv.restype = i64
        lib.or_floordiv.argtypes = [i64, i64]
        lib.or_lsh_key.restype = u32
        lib.or_lsh_key.argtypes = [vp, u32, u32, vp, vp, i32, u32]
        lib.or_build_index.argtypes = [vp, u32, u64, u32, u32, vp, vp, i32, u32, vp, vp, ci]
        lib.or_ssd.restype = u32
        lib.or_ssd.argtypes = [vp, vp]
        lib.or_perm_idx.restype = u64
        lib.or_perm_idx.argtypes = [u64, u64]
        lib.or_apply_writes.argtypes = [vp, u64, u32, ci, u64, u32, u64, u64]
        lib.or_compute.argtypes = [vp, u64, u32, u32, u64, ci, u32, vp, ci]
        lib.or_collage.argtypes = [vp, u32, u32, u32, u32, u32, vp, vp, i32, vp, u32, u64,
                                   vp, vp, u64, u64, vp, ci]
        _lib = lib
    return _lib


def _p(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def threads_default():
    return os.cpu_count() or 1


# ---------------------------------------------------------------- O1 reads
def sm64(x):
    return int(_load().or_sm64(x & (2**64 - 1)))


def fnv_words(h, value_bytes: bytes):
    buf = np.frombuffer(bytes(value_bytes), dtype=np.uint8).copy()
    return int(_load().or_fnv_words(h, _p(buf), len(value_bytes)))


def uniform_off(nbytes, elem, seed, t, i):
    return int(_load().or_uniform_off(nbytes, elem, seed, t, i))


def divergent_off(nbytes, page, elem, seed, t, i):
    return int(_load().or_divergent_off(nbytes, page, elem, seed, t, i))


def read_seq(file: np.ndarray, span, unit, elem, nthreads, passes=1, copy=False, threads=None):
    """SEQ pattern. Returns the copied bytes (copy=True) or per-thread checksums."""
    threads = threads or threads_default()
    if copy:
        out = np.zeros(span, dtype=np.uint8)
        _load().or_read_seq(_p(file), span, unit, elem, nthreads, passes, _p(out), None, threads)
        return out
    ck = np.empty(nthreads, dtype=np.uint64)
    _load().or_read_seq(_p(file), span, unit, elem, nthreads, passes, None, _p(ck), threads)
    return ck


def read_uniform(file: np.ndarray, nbytes, elem, nthreads, reads, seed, threads=None):
    ck = np.empty(nthreads, dtype=np.uint64)
    _load().or_read_uniform(_p(file), nbytes, elem, nthreads, reads, seed, _p(ck),
                            threads or threads_default())
    return ck


def read_divergent(file: np.ndarray, nbytes, page, elem, nthreads, reads, seed, threads=None):
    ck = np.empty(nthreads, dtype=np.uint64)
    _load().or_read_divergent(_p(file), nbytes, page, elem, nthreads, reads, seed, _p(ck),
                              threads or threads_default())
    return ck


def offsets(pattern, nbytes, elem, nthreads, reads, seed, page=0):
    """uint64[nthreads, reads]: the offset of read i of thread t (pattern
    1 = UNIFORM over nbytes, 2 = DIVERGENT with pattern page size `page`)."""
    out = np.empty((nthreads, reads), dtype=np.uint64)
    _load().or_offsets(pattern, nbytes, page, elem, seed, nthreads, reads, _p(out))
    return out


def perm_idx(k, M):
    return int(_load().or_perm_idx(k, M))


def apply_writes(file: np.ndarray, elem, pattern, nthreads=0, reads=0, span=None, seed=0):
    """The file after the write benchmark's stores (a new array)."""
    out = file.copy()
    span = file.nbytes if span is None else span
    _load().or_apply_writes(_p(out), file.nbytes, elem, pattern, nthreads, reads, span, seed)
    return out


def compute(file: np.ndarray, span, unit, elem, nthreads, work, iters=0, threads=None):
    """Per-thread accumulators of the compute-intensity workloads (float64)."""
    acc = np.empty(nthreads, dtype=np.float64)
    _load().or_compute(_p(file), span, unit, elem, nthreads, work, iters, _p(acc),
                       threads or threads_default())
    return acc


# ---------------------------------------------------------------- O3 collage
def block_hist(img: np.ndarray, b: int) -> np.ndarray:
    H, W, _ = img.shape
    h = np.empty(768, dtype=np.uint32)
    _load().or_block_hist(_p(np.ascontiguousarray(img)), W, H, b, _p(h))
    return h


def floordiv(a, b):
    return int(_load().or_floordiv(a, b))


def lsh_key(hist, t, proj, bias, w, bucket_bits):
    L, K = bias.shape
    hist = np.ascontiguousarray(hist, dtype=np.uint32)
    proj = np.ascontiguousarray(proj, dtype=np.int16)
    bias = np.ascontiguousarray(bias, dtype=np.int32)
    return int(_load().or_lsh_key(_p(hist), t, K, _p(proj), _p(bias), w, bucket_bits))


def build_index(file: np.ndarray, rec_stride, n, proj, bias, w, bucket_bits, threads=None):
    """Returns (offsets uint32[L, B+1], ids uint32[L, N])."""
    L, K = bias.shape
    B = 1 << bucket_bits
    offsets = np.empty((L, B + 1), dtype=np.uint32)
    ids = np.empty((L, n), dtype=np.uint32)
    proj = np.ascontiguousarray(proj, dtype=np.int16)
    bias = np.ascontiguousarray(bias, dtype=np.int32)
    _load().or_build_index(_p(file), rec_stride, n, L, K, _p(proj), _p(bias), w, bucket_bits,
                           _p(offsets), _p(ids), threads or threads_default())
    return offsets, ids


def ssd(a, b):
    a = np.ascontiguousarray(a, dtype=np.uint32)
    b = np.ascontiguousarray(b, dtype=np.uint32)
    return int(_load().or_ssd(_p(a), _p(b)))


def collage(img, proj, bias, w, bucket_bits, file, rec_stride, n, offsets, ids, b0=0, nb=None,
            threads=None):
    """Returns winners uint32[nb, 2] = (image index, squared distance)."""
    H, W, _ = img.shape
    L, K = bias.shape
    total = (W // 32) * (H // 32)
    nb = total - b0 if nb is None else nb
    out = np.empty((nb, 2), dtype=np.uint32)
    proj = np.ascontiguousarray(proj, dtype=np.int16)
    bias = np.ascontiguousarray(bias, dtype=np.int32)
    _load().or_collage(_p(np.ascontiguousarray(img)), W, H, L, K, bucket_bits, _p(proj),
                       _p(bias), w, _p(file), rec_stride, n, _p(offsets), _p(ids), b0, nb,
                       _p(out), threads or threads_default())
    return out
