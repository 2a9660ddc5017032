"""Multi-GPU collage on the CUDA path, checked
against the oracle running on its own bucket index:

* ap_collage_mgpu / ap_mgpu_* (C ABI, one process driving G partitions): the
  partitions' kernels fold their winners into the root's array with
  system-scope atomics; G partitions on repeated device ids exercise the same
  code on a one-GPU box;
* one process per rank (two processes sharing cuda:0, gloo): the fused path
  (mgpu.SharedWinners: CUDA IPC + AP_COLLAGE_ACCUMULATE | AP_COLLAGE_SYSTEM)
  and the collective baselines (mgpu.gather_winners, mgpu.reduce_winners_min)
  on winners the GPU produced."""
import os
import socket

import numpy as np
import pytest
import torch

import oracle
import synth
from helpers import make_records

pytestmark = pytest.mark.gpu

N, STRIDE, W_, H_, L, K, BB, WIDTH = 3000, 4096, 256, 192, 4, 5, 8, 2500


def _inputs(seed=51):
    recs = make_records(N, STRIDE, seed)
    proj, bias = synth.make_lsh_params(L, K, WIDTH, seed=seed + 1)
    img, _, _ = synth.make_target(W_, H_, N, ds_seed=seed, seed=seed + 2, pool=32,
                                  copy_permille=100)
    return recs, proj, bias, img


def _want(recs, proj, bias, img):
    o_off, o_ids = oracle.build_index(recs, STRIDE, N, proj, bias, WIDTH, BB)
    return oracle.collage(img, proj, bias, WIDTH, BB, recs, STRIDE, N, o_off, o_ids)


@pytest.mark.parametrize("partition", [0, 1, 2])  # AP_PART_BLOCKS / _RECORDS / _UNITS
@pytest.mark.parametrize("G", [1, 2, 3])
def test_collage_mgpu_c_abi(ap, partition, G):
    recs, proj, bias, img = _inputs()
    want = _want(recs, proj, bias, img)
    nb = (W_ // 32) * (H_ // 32)
    inp = ap.mgpu_collage_in(img, W_, H_, proj, bias, WIDTH, BB, N, STRIDE, group=8,
                             schedule=ap.AP_SCHED_TABLE, id_chunks=2, partition=partition)
    win = np.zeros((nb, 2), dtype=np.uint32)
    rep = ap.ap_collage_mgpu([0] * G, recs, 60, 4096, inp, win)
    assert rep["device_error"] == 0
    assert np.array_equal(win, want)
    assert len(rep["part_seconds"]) == G and rep["seconds"] > 0
    assert all(m > 0 for m in rep["major"])


def test_mgpu_context_repeats_and_reuploads(ap):
    """A context runs several cold steps; a changed target is re-uploaded."""
    recs, proj, bias, img = _inputs(seed=61)
    nb = (W_ // 32) * (H_ // 32)
    m = ap.ap_mgpu_create([0, 0], recs, 50, 4096)
    try:
        for step in range(3):
            tgt = img if step < 2 else np.ascontiguousarray(img[::-1])
            inp = ap.mgpu_collage_in(tgt, W_, H_, proj, bias, WIDTH, BB, N, STRIDE, group=4,
                                     schedule=ap.AP_SCHED_TABLE, partition=ap.AP_PART_RECORDS)
            win = np.zeros((nb, 2), dtype=np.uint32)
            rep = ap.ap_mgpu_collage(m, inp, win)
            assert rep["device_error"] == 0
            assert np.array_equal(win, _want(recs, proj, bias, tgt))
        with pytest.raises(ap.APError):  # records partition needs a per-table schedule
            ap.ap_mgpu_collage(m, ap.mgpu_collage_in(img, W_, H_, proj, bias, WIDTH, BB, N,
                                                     STRIDE, schedule=ap.AP_SCHED_LSH,
                                                     partition=ap.AP_PART_RECORDS), win)
    finally:
        ap.ap_mgpu_destroy(m)


def test_accumulate_flag_folds_partitions(ap):
    """ap_collage_in.flags = AP_COLLAGE_ACCUMULATE: block ranges and record
    slices of several calls (two caches) fold into one winners array."""
    recs, proj, bias, img = _inputs(seed=71)
    want = _want(recs, proj, bias, img)
    dev = torch.device("cuda:0")
    nb = (W_ // 32) * (H_ // 32)
    caches = [ap.ap_cache_create(40, 4096) for _ in range(2)]
    try:
        regs = [ap.ap_mmap(c, recs) for c in caches]
        B1 = (1 << BB) + 1
        off = torch.zeros((L, B1), dtype=torch.int32, device=dev)
        ids = torch.zeros((L, N), dtype=torch.int32, device=dev)
        pd, bd = torch.from_numpy(proj).to(dev), torch.from_numpy(bias).to(dev)
        ap.ap_lsh_build_index(caches[0], regs[0], N, STRIDE, L, K, BB, WIDTH, pd, bd, off, ids)
        tgt = torch.from_numpy(img).to(dev)
        for sched in (ap.AP_SCHED_NATURAL, ap.AP_SCHED_LSH, ap.AP_SCHED_TABLE):
            win = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
            ap.ap_winners_init(win, nb)
            for g in range(2):
                b0, b1 = g * nb // 2, (g + 1) * nb // 2
                inp = ap.collage_in(tgt, W_, H_, pd, bd, WIDTH, BB, off, ids, N, STRIDE, group=2,
                                    block_begin=b0, block_count=b1 - b0, schedule=sched,
                                    flags=ap.AP_COLLAGE_ACCUMULATE)
                ap.ap_collage_run(caches[g], regs[g], inp, win[b0:b1])
            torch.cuda.synchronize()
            assert np.array_equal(win.cpu().numpy().view(np.uint32), want), sched
        win = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
        ap.ap_winners_init(win, nb)
        for g in range(2):
            inp = ap.collage_in(tgt, W_, H_, pd, bd, WIDTH, BB, off, ids, N, STRIDE, group=8,
                                schedule=ap.AP_SCHED_TABLE, id_begin=g * N // 2,
                                id_end=(g + 1) * N // 2,
                                flags=ap.AP_COLLAGE_ACCUMULATE | ap.AP_COLLAGE_SYSTEM)
            ap.ap_collage_run(caches[g], regs[g], inp, win)
        torch.cuda.synchronize()
        assert np.array_equal(win.cpu().numpy().view(np.uint32), want)
        for c, r in zip(caches, regs):
            assert ap.ap_last_device_error(c) == 0
            ap.ap_munmap(c, r)
    finally:
        for c in caches:
            ap.ap_cache_destroy(c)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_worker(rank, world, port, q):
    import torch.distributed as dist

    import paper_conf_isca_shaharbs16_b200 as ap
    from paper_conf_isca_shaharbs16_b200 import mgpu
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    recs, proj, bias, img = _inputs()
    nb = (W_ // 32) * (H_ // 32)
    cache = ap.ap_cache_create(60, 4096)
    r = ap.ap_mmap(cache, recs)
    off = torch.zeros((L, (1 << BB) + 1), dtype=torch.int32, device=dev)
    ids = torch.zeros((L, N), dtype=torch.int32, device=dev)
    pd, bd = torch.from_numpy(proj).to(dev), torch.from_numpy(bias).to(dev)
    ap.ap_lsh_build_index(cache, r, N, STRIDE, L, K, BB, WIDTH, pd, bd, off, ids)
    tgt = torch.from_numpy(img).to(dev)
    out = {}
    # fused: every rank folds its record slice into rank 0's array (CUDA IPC)
    sw = mgpu.SharedWinners(ap, nb, rank, world, dist, dev)
    for part in ("records", "blocks"):
        sw.begin()
        if part == "records":
            i0, i1 = mgpu.id_range(N, rank, world)
            inp = ap.collage_in(tgt, W_, H_, pd, bd, WIDTH, BB, off, ids, N, STRIDE, group=8,
                                id_begin=i0, id_end=i1,
                                flags=ap.AP_COLLAGE_ACCUMULATE | ap.AP_COLLAGE_SYSTEM)
            ap.ap_collage_run(cache, r, inp, sw.ptr())
        else:
            b0, b1 = mgpu.block_range(nb, rank, world)
            inp = ap.collage_in(tgt, W_, H_, pd, bd, WIDTH, BB, off, ids, N, STRIDE, group=4,
                                block_begin=b0, block_count=b1 - b0, schedule=ap.AP_SCHED_LSH,
                                flags=ap.AP_COLLAGE_ACCUMULATE | ap.AP_COLLAGE_SYSTEM)
            ap.ap_collage_run(cache, r, inp, sw.ptr(b0))
        sw.end()
        if rank == 0:
            out["fused_" + part] = sw.result.cpu().numpy().view(np.uint32).copy()
    sw.close()
    # collective baselines on GPU-produced partials
    b0, b1 = mgpu.block_range(nb, rank, world)
    part = torch.zeros((b1 - b0, 2), dtype=torch.int32, device=dev)
    ap.ap_collage_run(cache, r, ap.collage_in(tgt, W_, H_, pd, bd, WIDTH, BB, off, ids, N,
                                              STRIDE, group=8, block_begin=b0,
                                              block_count=b1 - b0), part)
    full = mgpu.gather_winners(part, rank, world, dist, nb)
    if rank == 0:
        out["gather_blocks"] = full.cpu().numpy().view(np.uint32).copy()
    u0, u1 = mgpu.unit_range(L * nb, rank, world)
    part = torch.zeros((nb, 2), dtype=torch.int32, device=dev)
    ap.ap_collage_run(cache, r, ap.collage_in(tgt, W_, H_, pd, bd, WIDTH, BB, off, ids, N,
                                              STRIDE, group=8, unit_begin=u0,
                                              unit_count=u1 - u0), part)
    red = mgpu.reduce_winners_min(part, rank, world, dist)
    if rank == 0:
        out["reduce_units"] = red.cpu().numpy().view(np.uint32).copy()
    torch.cuda.synchronize()
    out["err"] = ap.ap_last_device_error(cache)
    ap.ap_munmap(cache, r)
    ap.ap_cache_destroy(cache)
    q.put((rank, out))
    dist.barrier()
    dist.destroy_process_group()


def test_one_process_per_rank_fused_and_collectives():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    world = 2
    procs = [ctx.Process(target=_rank_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    want = _want(*_inputs())
    assert all(got[r]["err"] == 0 for r in range(world))
    for k in ("fused_records", "fused_blocks", "gather_blocks", "reduce_units"):
        assert np.array_equal(got[0][k], want), k
