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


def _load_runs(lines):
    """(index, count) of each run of 16-B loads: the loads issued from one
    LDG.E.128 until the next branch (other instructions may interleave; a
    branch ends the straight-line stretch the loads are in flight across)."""
    runs, n = [], 0
    while n < len(lines):
        if "LDG.E.128" in lines[n]:
            k, cnt = n, 0
            while k < len(lines) and not re.search(r"\b(BRA|EXIT|CALL|RET|BSYNC)\b", lines[k]):
                cnt += "LDG.E.128" in lines[k]
                k += 1
            runs.append((n, cnt))
            n = k + 1
        else:
            n += 1
    return runs


@pytest.mark.parametrize("aptr", ["Lb1", "Lb0"])
def test_seq_tile_keeps_16_loads_in_flight(ap, aptr):
    """k_seq<uint4, apointer|raw>: the 16-B tile issues its 16 loads in one
    straight-line stretch, and no local-memory spill sits inside that tile."""
    lines = _function(_sass(ap), r"k_seqI5uint4" + aptr + "EEE")
    runs = _load_runs(lines)
    full = [(n, ln) for n, ln in runs if ln >= 16]
    assert full, runs[:12]
    first = full[0][0]
    tile = lines[first:first + 16 * 8]
    assert sum("STL" in ln or "LDL" in ln for ln in tile) <= 2


def test_per_access_deref_keeps_values_in_registers(ap):
    """k_seq_deref<uint4, apointer>: the per-access loop keeps the values of
    the accesses in flight in registers across the (out-of-line, ABI) fault
    path -- no STL right after a 16-B load (a spill there makes every
    access wait for its data before the next one is issued)."""
    lines = _function(_sass(ap), r"k_seq_derefI5uint4Lb1ELb0EEE")
    for i, ln in enumerate(lines):
        if "LDG.E.128" in ln:
            after = lines[i + 1:i + 6]
            assert not any(re.match(r"(@\S+\s+)?STL", a) for a in after), (ln, after)
