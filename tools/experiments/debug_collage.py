"""Debug driver: one collage run with a short watchdog, then stats/invariants."""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
sys.path.insert(0, "tests")
import oracle  # noqa: E402
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402
from helpers import check_invariants, make_records  # noqa: E402

group = int(sys.argv[1]) if len(sys.argv) > 1 else 4
frames = int(sys.argv[2]) if len(sys.argv) > 2 else 48
dev = torch.device("cuda:0")
n, stride, w, bb, L, K = 4096, 4096, 2500, 9, 4, 6
W, H = 512, 256
recs = make_records(n, stride, 21)
proj, bias = synth.make_lsh_params(L, K, w, seed=22)
img, src, is_copy = synth.make_target(W, H, n, ds_seed=21, seed=23, pool=32, copy_permille=100)
cache = ap.ap_cache_create(frames, 4096)
ap.ap_cache_set_tuning(cache, 1, 64, 3000)
r = ap.ap_mmap(cache, recs)
off = torch.zeros((L, (1 << bb) + 1), dtype=torch.int32, device=dev)
ids = torch.zeros((L, n), dtype=torch.int32, device=dev)
pd, bd = torch.from_numpy(proj).to(dev), torch.from_numpy(bias).to(dev)
ap.ap_lsh_build_index(cache, r, n, stride, L, K, bb, w, pd, bd, off, ids)
tgt = torch.from_numpy(img).to(dev)
nb = (W // 32) * (H // 32)
win = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
t0 = time.time()
ap.ap_collage_run(cache, r, ap.collage_in(tgt, W, H, pd, bd, w, bb, off, ids, n, group=group), win)
torch.cuda.synchronize()
print("kernel s", time.time() - t0, "err", ap.ap_last_device_error(cache))
print(ap.ap_cache_stats(cache))
want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, off.cpu().numpy().view(np.uint32),
                      ids.cpu().numpy().view(np.uint32))
got = win.cpu().numpy().view(np.uint32)
print("mismatch blocks", int((got != want).any(axis=1).sum()), "of", nb)
print("invariants", check_invariants(ap, cache, [r], frames)[:5])
