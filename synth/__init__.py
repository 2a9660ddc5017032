"""Seeded synthetic input generators.

Shared by the CUDA path's drivers and by the tests that feed the oracle. It
holds none of the method's arithmetic (see synth.c's header): it draws
counter-based random numbers and lays them out like the paper's workloads
(PAPER.md:363-371 microbenchmark file; PAPER.md:411-419 collage dataset,
target image and LSH draws).
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libsynth.so")
_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `make` (or __graft_entry__.build())")
        lib = ctypes.CDLL(_LIB_PATH)
        u64, u32, i32, vp = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int32, ctypes.c_void_p
        lib.synth_sm64.restype = u64
        lib.synth_sm64.argtypes = [u64]
        lib.synth_file.argtypes = [vp, u64, u64]
        lib.synth_tile_pixels.argtypes = [u64, u64, vp]
        lib.synth_records.argtypes = [vp, u64, u64, u32, u64]
        lib.synth_target.argtypes = [vp, u32, u32, u64, u64, u64, u32, u32, vp, vp]
        lib.synth_lsh_params.argtypes = [vp, vp, u32, u32, i32, u64]
        _lib = lib
    return _lib


def _ptr(a):
    return ctypes.c_void_p(a.ctypes.data)


def sm64(x: int) -> int:
    return int(_load().synth_sm64(ctypes.c_uint64(x & (2**64 - 1))))


def fill_file(buf: np.ndarray, seed: int) -> np.ndarray:
    """Fill a uint8 buffer in place with the microbenchmark file contents."""
    assert buf.dtype == np.uint8 and buf.flags.c_contiguous
    _load().synth_file(_ptr(buf), buf.nbytes, seed)
    return buf


def make_file(nbytes: int, seed: int) -> np.ndarray:
    return fill_file(np.empty(nbytes, dtype=np.uint8), seed)


def tile_pixels(seed: int, i: int) -> np.ndarray:
    px = np.empty(3072, dtype=np.uint8)
    _load().synth_tile_pixels(seed, i, _ptr(px))
    return px


def fill_records(buf: np.ndarray, first: int, count: int, rec_stride: int, seed: int):
    """Write records [first, first+count) into buf (buf[0] = record `first`)."""
    assert buf.dtype == np.uint8 and buf.nbytes >= count * rec_stride
    _load().synth_records(_ptr(buf), first, count, rec_stride, seed)
    return buf


def make_records(n: int, rec_stride: int, seed: int) -> np.ndarray:
    return fill_records(np.empty(n * rec_stride, dtype=np.uint8), 0, n, rec_stride, seed)


def make_target(W: int, H: int, n_records: int, ds_seed: int, seed: int, pool: int = 256,
                copy_permille: int = 50):
    """Returns (img uint8[H, W, 3], src int64[blocks], is_copy uint8[blocks])."""
    assert W % 32 == 0 and H % 32 == 0
    img = np.empty((H, W, 3), dtype=np.uint8)
    nb = (W // 32) * (H // 32)
    src = np.empty(nb, dtype=np.int64)
    is_copy = np.empty(nb, dtype=np.uint8)
    _load().synth_target(_ptr(img), W, H, n_records, ds_seed, seed, pool, copy_permille,
                         _ptr(src), _ptr(is_copy))
    return img, src, is_copy


def make_lsh_params(L: int, K: int, w: int, seed: int):
    """Returns (proj int16[L, K, 768], bias int32[L, K])."""
    proj = np.empty((L, K, 768), dtype=np.int16)
    bias = np.empty((L, K), dtype=np.int32)
    _load().synth_lsh_params(_ptr(proj), _ptr(bias), L, K, w, seed)
    return proj, bias
