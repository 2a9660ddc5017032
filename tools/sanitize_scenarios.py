"""Small scenarios for compute-sanitizer (memcheck / racecheck / synccheck):
every fault-path branch (minor, major, eviction, exhaustion back-off,
divergent groups, partial warps, tiles straddling pages) on tiny inputs,
each checked against the oracle so a sanitizer run is also a parity run."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
sys.path.insert(0, "tests")
import oracle  # noqa: E402
import paper_conf_isca_shaharbs16_b200 as ap  # noqa: E402
import synth  # noqa: E402
from helpers import check_invariants, make_file, make_records  # noqa: E402

dev = torch.device("cuda:0")
ok = True


def check(name, cond):
    global ok
    print(f"{name}: {'ok' if cond else 'FAIL'}", flush=True)
    ok &= bool(cond)


f = make_file((1 << 20) + 4096 * 3 + 48, 1)
for frames, policy in ((2, 0), (8, 1)):
    c = ap.ap_cache_create(frames, 4096)
    ap.ap_cache_set_policy(c, policy, 3)
    r = ap.ap_mmap(c, f)
    n = f.nbytes
    out = torch.zeros(n, dtype=torch.uint8, device=dev)
    ap.ap_bench_read(c, r, ap.bench_cfg(ap.AP_SEQ, 16, 2, 64, unit_bytes=4096, out_copy=True,
                                        span_bytes=n), out)
    torch.cuda.synchronize()
    whole = n // 16 * 16
    check(f"seq copy frames={frames}", np.array_equal(out.cpu().numpy()[:whole], f[:whole]))
    ck = torch.zeros(256, dtype=torch.int64, device=dev)
    ap.ap_bench_read(c, r, ap.bench_cfg(ap.AP_UNIFORM, 4, 2, 128, reads_per_thread=3, seed=5), ck)
    torch.cuda.synchronize()
    check(f"uniform frames={frames}", np.array_equal(ck.cpu().numpy().view(np.uint64),
                                                     oracle.read_uniform(f, n, 4, 256, 3, 5)))
    nd = 64 * 4096
    ap.ap_bench_read(c, r, ap.bench_cfg(ap.AP_DIVERGENT, 16, 2, 128, reads_per_thread=2,
                                        page_bytes=4096, seed=9), ck)
    torch.cuda.synchronize()
    check(f"divergent frames={frames}", np.array_equal(
        ck.cpu().numpy().view(np.uint64), oracle.read_divergent(f, n, 4096, 16, 256, 2, 9)))
    for acc in (ap.AP_ACCESS_DEREF, ap.AP_ACCESS_RANGE):
        ck2 = torch.zeros(128, dtype=torch.int64, device=dev)
        ap.ap_bench_read(c, r, ap.bench_cfg(ap.AP_SEQ, 16, 1, 128, unit_bytes=4096, access=acc), ck2)
        torch.cuda.synchronize()
        check(f"seq access={acc} frames={frames}", np.array_equal(
            ck2.cpu().numpy().view(np.uint64), oracle.read_seq(f, n, 4096, 16, 128, 1)))
    check(f"invariants frames={frames}", check_invariants(ap, c, [r], frames) == [])
    check(f"device error frames={frames}", ap.ap_last_device_error(c) == 0)
    ap.ap_munmap(c, r)
    ap.ap_cache_destroy(c)

# collage: groups 1/2/4 over a 12-frame cache, both schedules, unaligned-free
n, stride, w, bb = 512, 4096, 2500, 6
recs = make_records(n, stride, 3)
proj, bias = synth.make_lsh_params(2, 4, w, seed=4)
img, _, _ = synth.make_target(128, 64, n, ds_seed=3, seed=5, pool=4, copy_permille=100)
c = ap.ap_cache_create(12, 4096)
r = ap.ap_mmap(c, recs)
off = torch.zeros((2, (1 << bb) + 1), dtype=torch.int32, device=dev)
ids = torch.zeros((2, n), dtype=torch.int32, device=dev)
pd, bd = torch.from_numpy(proj).to(dev), torch.from_numpy(bias).to(dev)
ap.ap_lsh_build_index(c, r, n, stride, 2, 4, bb, w, pd, bd, off, ids)
o_off, o_ids = oracle.build_index(recs, stride, n, proj, bias, w, bb)
check("index", np.array_equal(off.cpu().numpy().view(np.uint32), o_off))
want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, o_off, o_ids)
tgt = torch.from_numpy(img).to(dev)
for g in (1, 2, 4):
    for sch in (0, 1):
        win = torch.zeros((8, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(c, r, ap.collage_in(tgt, 128, 64, pd, bd, w, bb, off, ids, n, group=g,
                                              schedule=sch), win)
        torch.cuda.synchronize()
        check(f"collage group={g} schedule={sch}",
              np.array_equal(win.cpu().numpy().view(np.uint32), want))
check("collage invariants", check_invariants(ap, c, [r], 12) == [])
ap.ap_munmap(c, r)
ap.ap_cache_destroy(c)
# unaligned 3 KiB records (tiles straddle pages)
recs3 = make_records(n, 3072, 3)
c = ap.ap_cache_create(6, 4096)
r = ap.ap_mmap(c, recs3)
ap.ap_lsh_build_index(c, r, n, 3072, 2, 4, bb, w, pd, bd, off, ids)
o_off, o_ids = oracle.build_index(recs3, 3072, n, proj, bias, w, bb)
want = oracle.collage(img, proj, bias, w, bb, recs3, 3072, n, o_off, o_ids)
for g in (1, 4):
    win = torch.zeros((8, 2), dtype=torch.int32, device=dev)
    ap.ap_collage_run(c, r, ap.collage_in(tgt, 128, 64, pd, bd, w, bb, off, ids, n, 3072, group=g),
                      win)
    torch.cuda.synchronize()
    check(f"unaligned collage group={g}", np.array_equal(win.cpu().numpy().view(np.uint32), want))
check("unaligned invariants", check_invariants(ap, c, [r], 6) == [])
ap.ap_munmap(c, r)
ap.ap_cache_destroy(c)
# writable mappings: scattered stores with 3 frames (dirty write-back during
# the kernel), apointer-to-apointer copy with 4 frames
fw = make_file(1 << 20, 9)
want_w = oracle.apply_writes(fw, 4, 1, nthreads=256, reads=4, seed=3)
c = ap.ap_cache_create(3, 4096)
r = ap.ap_mmap_prot(c, fw, 3)
ap.ap_bench_write(c, r, ap.bench_cfg(ap.AP_UNIFORM, 4, 2, 128, reads_per_thread=4, seed=3))
torch.cuda.synchronize()
check("writes device error", ap.ap_last_device_error(c) == 0)
ap.ap_munmap(c, r)
check("writes reach the file", np.array_equal(fw, want_w))
src, dst = make_file(1 << 19, 10), make_file(1 << 19, 11)
r1 = ap.ap_mmap(c, src)
r2 = ap.ap_mmap_prot(c, dst, 3)
ap.ap_bench_copy(c, r1, r2, ap.bench_cfg(ap.AP_SEQ, 16, 2, 64, unit_bytes=4096))
torch.cuda.synchronize()
check("copy device error", ap.ap_last_device_error(c) == 0)
check("copy invariants", check_invariants(ap, c, [r1, r2], 3) == [])
ap.ap_munmap(c, r2)
ap.ap_munmap(c, r1)
check("copy reaches the file", np.array_equal(dst, src))
ap.ap_cache_destroy(c)
# per-table schedules with record-id windows and a record-id range (the
# by-records multi-GPU share), over a 12-frame cache
c = ap.ap_cache_create(12, 4096)
r = ap.ap_mmap(c, recs)
for sch in (2, 3):
    for kw in (dict(id_chunks=3), dict(id_chunks=2, id_begin=0, id_end=n // 2)):
        win = torch.zeros((8, 2), dtype=torch.int32, device=dev)
        ap.ap_collage_run(c, r, ap.collage_in(tgt, 128, 64, pd, bd, w, bb, off, ids, n, group=8,
                                              schedule=sch, **kw), win)
        torch.cuda.synchronize()
        if "id_end" in kw:
            win2 = torch.zeros((8, 2), dtype=torch.int32, device=dev)
            ap.ap_collage_run(c, r, ap.collage_in(tgt, 128, 64, pd, bd, w, bb, off, ids, n,
                                                  group=8, schedule=sch, id_begin=n // 2), win2)
            torch.cuda.synchronize()
            f = torch.tensor(-(1 << 63), dtype=torch.int64, device=dev)
            win = ((torch.minimum(win.view(torch.int64).view(-1) ^ f,
                                  win2.view(torch.int64).view(-1) ^ f)) ^ f).view(torch.int32).view(-1, 2)
        check(f"collage schedule={sch} {sorted(kw)}", np.array_equal(win.cpu().numpy().view(np.uint32), want))
check("windows invariants", check_invariants(ap, c, [r], 12) == [])
check("windows device error", ap.ap_last_device_error(c) == 0)
ap.ap_munmap(c, r)
ap.ap_cache_destroy(c)

# peer caches: two 3-frame caches that are each other's peer, reading at once
fp = make_file(32 * 4096, 4)
ca, cb = ap.ap_cache_create(3, 4096), ap.ap_cache_create(3, 4096)
ra, rb = ap.ap_mmap(ca, fp), ap.ap_mmap(cb, fp)
ap.ap_region_add_peer(ca, ra, cb, rb)
ap.ap_region_add_peer(cb, rb, ca, ra)
sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
cka = torch.zeros(128, dtype=torch.int64, device=dev)
ckb = torch.zeros(128, dtype=torch.int64, device=dev)
ap.ap_bench_read(ca, ra, ap.bench_cfg(ap.AP_UNIFORM, 4, 1, 128, reads_per_thread=4, seed=7), cka, sa)
ap.ap_bench_read(cb, rb, ap.bench_cfg(ap.AP_UNIFORM, 4, 1, 128, reads_per_thread=4, seed=8), ckb, sb)
torch.cuda.synchronize()
check("peers a", np.array_equal(cka.cpu().numpy().view(np.uint64), oracle.read_uniform(fp, fp.nbytes, 4, 128, 4, 7)))
check("peers b", np.array_equal(ckb.cpu().numpy().view(np.uint64), oracle.read_uniform(fp, fp.nbytes, 4, 128, 4, 8)))
check("peers invariants", check_invariants(ap, ca, [ra], 3) == [] and check_invariants(ap, cb, [rb], 3) == [])
# split-phase link styles
for acc in (ap.AP_ACCESS_AHEAD, ap.AP_ACCESS_PAIR):
    ck2 = torch.zeros(128, dtype=torch.int64, device=dev)
    ap.ap_bench_read(ca, ra, ap.bench_cfg(ap.AP_SEQ, 16, 1, 128, unit_bytes=4096, access=acc), ck2)
    torch.cuda.synchronize()
    check(f"seq access={acc} (peers on)", np.array_equal(
        ck2.cpu().numpy().view(np.uint64), oracle.read_seq(fp, fp.nbytes, 4096, 16, 128, 1)))
check("peers device error", ap.ap_last_device_error(ca) == 0 and ap.ap_last_device_error(cb) == 0)
ap.ap_region_clear_peers(ca, ra)
ap.ap_region_clear_peers(cb, rb)
ap.ap_munmap(ca, ra)
ap.ap_munmap(cb, rb)
ap.ap_cache_destroy(ca)
ap.ap_cache_destroy(cb)

# [r2] per-access dereference (deferred unlink at the next dereference) and the
# drop-behind policy, with frames scarce; Fig. 6 ADD (two pointers, the miss
# path releases the other one under pressure)
fd_ = make_file((1 << 20) + 4096 * 3 + 48, 2)
for frames, policy in ((3, ap.AP_POLICY_SEQUENTIAL), (5, ap.AP_POLICY_CLOCK)):
    c = ap.ap_cache_create(frames, 4096)
    ap.ap_cache_set_policy(c, policy)
    r = ap.ap_mmap(c, fd_)
    ck = torch.zeros(128, dtype=torch.int64, device=dev)
    ap.ap_bench_read(c, r, ap.bench_cfg(ap.AP_SEQ, 16, 1, 128, unit_bytes=4096,
                                        access=ap.AP_ACCESS_DEREF), ck)
    torch.cuda.synchronize()
    check(f"deref frames={frames} policy={policy}", np.array_equal(
        ck.cpu().numpy().view(np.uint64), oracle.read_seq(fd_, fd_.nbytes, 4096, 16, 128, 1)))
    check(f"deref invariants frames={frames}", check_invariants(ap, c, [r], frames) == [])
    ap.ap_munmap(c, r)
    ap.ap_cache_destroy(c)
# [r2] the C1 launch: page units from the work queue (AP_SEQ_QUEUE) under the
# drop-behind policy (pin kept across the fault, claim-first probe), fewer
# frames than warps
for frames in (3, 8):
    c = ap.ap_cache_create(frames, 4096)
    ap.ap_cache_set_policy(c, ap.AP_POLICY_SEQUENTIAL)
    r = ap.ap_mmap(c, fd_)
    outq = torch.zeros(fd_.nbytes, dtype=torch.uint8, device=dev)
    ap.ap_bench_read(c, r, ap.bench_cfg(ap.AP_SEQ_QUEUE, 16, 12, 32, unit_bytes=4096,
                                        out_copy=True, span_bytes=fd_.nbytes), outq)
    torch.cuda.synchronize()
    w = fd_.nbytes // 16 * 16
    check(f"queue frames={frames}", np.array_equal(outq.cpu().numpy()[:w], fd_[:w]))
    check(f"queue invariants frames={frames}", check_invariants(ap, c, [r], frames) == [])
    ap.ap_munmap(c, r)
    ap.ap_cache_destroy(c)
fa = make_file(1 << 21, 4)
c = ap.ap_cache_create(4, 4096)
r = ap.ap_mmap(c, fa)
acc = torch.zeros(64, dtype=torch.int64, device=dev)
ap.ap_bench_compute(c, r, "add", 16, 1, 64, 1 << 20, acc)
torch.cuda.synchronize()
want = oracle.compute(fa, 1 << 20, 4096, 16, 64, 0)
check("compute add frames=4", np.array_equal(acc.cpu().numpy().view(np.uint64).astype(np.float64),
                                              want))
check("compute add invariants", check_invariants(ap, c, [r], 4) == [])
ap.ap_munmap(c, r)
ap.ap_cache_destroy(c)

# [r2] multi-partition collage through the C ABI (three partitions on this
# GPU fold winners into one array with system-scope atomics)
nm = 600
recs_m = make_records(nm, 4096, 13)
proj_m, bias_m = synth.make_lsh_params(2, 4, 2500, seed=14)
img_m, _, _ = synth.make_target(128, 64, nm, ds_seed=13, seed=15, pool=8, copy_permille=100)
o_off_m, o_ids_m = oracle.build_index(recs_m, 4096, nm, proj_m, bias_m, 2500, 6)
want_m = oracle.collage(img_m, proj_m, bias_m, 2500, 6, recs_m, 4096, nm, o_off_m, o_ids_m)
for part in (ap.AP_PART_BLOCKS, ap.AP_PART_RECORDS):
    win_m = np.zeros(((128 // 32) * (64 // 32), 2), dtype=np.uint32)
    inp_m = ap.mgpu_collage_in(img_m, 128, 64, proj_m, bias_m, 2500, 6, nm, group=4,
                               partition=part)
    rep = ap.ap_collage_mgpu([0, 0, 0], recs_m, 5, 4096, inp_m, win_m)
    check(f"mgpu partition={part}", np.array_equal(win_m, want_m) and rep["device_error"] == 0)

print("ALL OK" if ok else "FAILURES")
sys.exit(0 if ok else 1)
