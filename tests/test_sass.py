"""Code-generation guards on the built library (CPU only: cuobjdump reads
the sm_100a SASS).  The hit path's performance depends on ptxas keeping a
whole 16-deep tile of 16-B loads in flight in the tiled SEQ kernel; an
unrelated change to the out-of-line fault path once made ptxas interleave
the tile with its consumption (9 loads in flight) and spill the checksum,
costing a third of the hit-mode bandwidth.  These checks catch that here,
before a GPU run."""
import os
import re
import shutil
import subprocess

import pytest

CUOBJDUMP = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"


def _sass(ap):
    from paper_conf_isca_shaharbs16_b200 import _lib
    if not os.path.exists(CUOBJDUMP):
        pytest.skip("cuobjdump not available")
    return subprocess.run([CUOBJDUMP, "-sass", _lib.LIB_PATH], capture_output=True,
                          text=True).stdout


def _function(sass, pattern):
    m = re.search(r"Function : (\S*" + pattern + r"\S*)", sass)
    assert m, pattern
    j = sass.find("Function : ", m.end())
    body = sass[m.start():j if j > 0 else None]
    return [re.sub(r"/\*[0-9a-f]+\*/", "", ln).split(";")[0].strip()
            for ln in body.splitlines() if re.search(r"/\*[0-9a-f]{4,}\*/", ln)]


@pytest.mark.parametrize("aptr", ["Lb1", "Lb0"])
def test_seq_tile_keeps_16_loads_in_flight(ap, aptr):
    """k_seq<uint4, apointer|raw>: the first 16-B tile issues 16 loads back to
    back, and no local-memory spill sits inside that tile."""
    lines = _function(_sass(ap), r"k_seqI5uint4" + aptr + "EEE")
    # runs of 16-B loads, allowing one other instruction between two loads
    runs, n = [], 0
    while n < len(lines):
        if "LDG.E.128" in lines[n]:
            k, cnt = n, 0
            while k < len(lines) and ("LDG.E.128" in lines[k] or
                                      (k + 1 < len(lines) and "LDG.E.128" in lines[k + 1]
                                       and "LDG.E.128" in lines[k - 1])):
                cnt += "LDG.E.128" in lines[k]
                k += 1
            runs.append((n, cnt))
            n = k
        else:
            n += 1
    full = [(n, ln) for n, ln in runs if ln >= 16]
    assert full, runs[:12]
    # the tile loop (the first full-depth run) has no spill traffic in it
    first = full[0][0]
    tile = lines[first:first + 16 * 8]
    assert sum("STL" in ln or "LDL" in ln for ln in tile) <= 2
