"""Host-side checks of the boundary (no GPU needed): the C-ABI library loads,
exports every function include/ap.h declares, and its error paths that need no
device behave as documented."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "ap.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ap_[a-z_]+)\s*\(", src)))


def test_header_declares_the_paper_boundary():
    names = _declared()
    for n in ("ap_cache_create", "ap_cache_destroy", "ap_mmap", "ap_munmap", "ap_bench_read",
              "ap_collage_run", "ap_lsh_build_index", "ap_cache_stats", "ap_cache_reset"):
        assert n in names


def test_library_exports_every_declared_symbol(ap):
    from paper_conf_isca_shaharbs16_b200 import _lib
    L = ctypes.CDLL(_lib.LIB_PATH)
    missing = [n for n in _declared() if not hasattr(L, n)]
    assert missing == []
    assert set(_lib.EXPORTED) == set(_declared())


def test_library_is_built_for_sm100a(ap):
    import subprocess
    from paper_conf_isca_shaharbs16_b200 import _lib
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _lib.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_strerror_and_version(ap):
    assert ap.ap_strerror(0) == "ok"
    assert "region" in ap.ap_strerror(-6)
    assert ap.ap_strerror(-123) == "unknown error"
    assert "sm_100a" in ap.ap_version()


def test_invalid_arguments_rejected_without_a_device(ap):
    from paper_conf_isca_shaharbs16_b200 import _lib
    L = _lib.lib()
    h = ctypes.c_void_p()
    # page size not a power of two / zero frames: rejected before touching CUDA
    assert L.ap_cache_create(16, 5000, 0, ctypes.byref(h)) == _lib.AP_EINVAL
    assert L.ap_cache_create(0, 4096, 0, ctypes.byref(h)) == _lib.AP_EINVAL
    assert L.ap_cache_create(16, 4096, 0, None) == _lib.AP_EINVAL
    assert L.ap_cache_destroy(None) == _lib.AP_EINVAL
    assert L.ap_mmap(None, None, 0, None) == _lib.AP_EINVAL
    assert L.ap_bench_read(None, 0, None, None, None) == _lib.AP_EINVAL
    assert L.ap_collage_run(None, 0, None, None, None) == _lib.AP_EINVAL
    with pytest.raises(_lib.APError):
        ap.ap_cache_create(0, 4096)


def test_product_never_imports_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_isca_shaharbs16_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dp, f)).read()
                assert "oracle" not in txt.replace("PAPER", ""), f
