"""Pick the LSH bucket width w for the synthetic collage dataset (DESIGN.md
R-A5: median non-empty bucket 32-256 ids at the full N, max < 64x median).
Calls only oracle/ and synth/ (a committed script, per the oracle rules)."""
import sys

import numpy as np

sys.path.insert(0, ".")
import oracle  # noqa: E402
import synth  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 200_000
full = int(sys.argv[2]) if len(sys.argv) > 2 else 1 << 20
bb = int(sys.argv[3]) if len(sys.argv) > 3 else 14
recs = synth.make_records(n, 4096, 21)
for w in [int(x) for x in (sys.argv[4].split(",") if len(sys.argv) > 4 else "20000,50000,100000,200000,400000".split(","))]:
    proj, bias = synth.make_lsh_params(1, 8, w, seed=22)
    off, ids = oracle.build_index(recs, 4096, n, proj, bias, w, bb)
    sizes = np.diff(off[0].astype(np.int64))
    nz = sizes[sizes > 0] * (full / n)
    print(f"w={w:6d} nonempty={len(nz):6d} median={np.median(nz):8.1f} p99={np.percentile(nz, 99):9.1f} "
          f"max={nz.max():9.1f} mean_cands_per_query~{(sizes.astype(float) ** 2).sum() / n * full / n:9.1f}")
