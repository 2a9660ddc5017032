"""The N>1 collage path on CPU: two gloo ranks each compute their block range
(with the oracle -- the GPU kernels are covered by the gpu tests) and gather
the winners with paper_conf_isca_shaharbs16_b200.mgpu; rank 0 must hold
exactly the single-process answer."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_isca_shaharbs16_b200 import mgpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _setup():
    n, stride, w, bb = 1500, 4096, 2500, 8
    recs = synth.make_records(n, stride, 7)
    proj, bias = synth.make_lsh_params(3, 5, w, seed=8)
    img, _, _ = synth.make_target(224, 96, n, ds_seed=7, seed=9, pool=16, copy_permille=100)
    off, ids = oracle.build_index(recs, stride, n, proj, bias, w, bb, threads=1)
    return n, stride, w, bb, recs, proj, bias, img, off, ids


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n, stride, w, bb, recs, proj, bias, img, off, ids = _setup()
    nb = (224 // 32) * (96 // 32)
    b0, b1 = mgpu.block_range(nb, rank, world)
    mine = oracle.collage(img, proj, bias, w, bb, recs, stride, n, off, ids, b0=b0, nb=b1 - b0,
                          threads=1)
    full = mgpu.gather_winners(torch.from_numpy(mine.view(np.int32)), rank, world, dist, nb)
    if rank == 0:
        q.put(full.numpy().view(np.uint32).copy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_partitioned_collage_gathers_the_whole_answer(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    n, stride, w, bb, recs, proj, bias, img, off, ids = _setup()
    want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, off, ids, threads=1)
    assert np.array_equal(got, want)


def test_block_ranges_cover_exactly():
    for nb in (1, 7, 21, 1024, 65536):
        for world in (1, 2, 3, 8):
            rs = [mgpu.block_range(nb, r, world) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == nb
            assert all(rs[i][1] == rs[i + 1][0] for i in range(world - 1))
            assert max(b - a for a, b in rs) - min(b - a for a, b in rs) <= 1


def _worker_tables(rank, world, port, q):
    """Bucket partition (AP_SCHED_TABLE across ranks): rank r owns the units of
    tables t = r, r + world, ...; its partial winners (oracle over those
    tables' buckets only) are combined by the unsigned 64-bit MIN reduction."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n, stride, w, bb, recs, proj, bias, img, off, ids = _setup()
    mine_off = off.copy()
    for t in range(off.shape[0]):
        if t % world != rank:
            mine_off[t] = 0  # every bucket of a table this rank does not own is empty
    part = oracle.collage(img, proj, bias, w, bb, recs, stride, n, mine_off, ids, threads=1)
    full = mgpu.reduce_winners_min(torch.from_numpy(part.view(np.int32).copy()), rank, world, dist)
    if rank == 0:
        q.put(full.numpy().view(np.uint32).copy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_bucket_partition_min_reduces_to_the_whole_answer(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_tables, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    n, stride, w, bb, recs, proj, bias, img, off, ids = _setup()
    want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, off, ids, threads=1)
    assert np.array_equal(got, want)
    # some block must have had candidates in only part of the tables, else
    # the reduction was not exercised
    assert (want[:, 0] != 0xFFFFFFFF).any()


def test_unit_ranges_cover_exactly():
    for nu in (1, 9, 4096, 262144):
        for world in (1, 2, 3, 8):
            rs = [mgpu.unit_range(nu, r, world) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == nu
            assert all(rs[i][1] == rs[i + 1][0] for i in range(world - 1))


def _restrict_index(off, ids, i0, i1):
    """The bucket CSR with every id outside [i0, i1) dropped (test-side
    marshalling of the by-records split; the oracle itself is unchanged)."""
    off_r, ids_r = np.zeros_like(off), np.zeros_like(ids)
    for t in range(off.shape[0]):
        k = 0
        for b in range(off.shape[1] - 1):
            off_r[t, b] = k
            seg = ids[t, off[t, b]:off[t, b + 1]]
            seg = seg[(seg >= i0) & (seg < i1)]
            ids_r[t, k:k + seg.size] = seg
            k += seg.size
        off_r[t, -1] = k
    return off_r, ids_r


def _worker_records(rank, world, port, q):
    """By-records partition: rank r sees only candidates whose record id is
    in mgpu.id_range(N, r, world); the MIN reduction gives the whole answer."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n, stride, w, bb, recs, proj, bias, img, off, ids = _setup()
    i0, i1 = mgpu.id_range(n, rank, world)
    off_r, ids_r = _restrict_index(off, ids, i0, i1)
    part = oracle.collage(img, proj, bias, w, bb, recs, stride, n, off_r, ids_r, threads=1)
    full = mgpu.reduce_winners_min(torch.from_numpy(part.view(np.int32).copy()), rank, world, dist)
    if rank == 0:
        q.put(full.numpy().view(np.uint32).copy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_record_partition_min_reduces_to_the_whole_answer(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_records, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    n, stride, w, bb, recs, proj, bias, img, off, ids = _setup()
    want = oracle.collage(img, proj, bias, w, bb, recs, stride, n, off, ids, threads=1)
    assert np.array_equal(got, want)


def test_id_ranges_cover_exactly():
    for n in (1, 9, 1500, 10_000_000):
        for world in (1, 2, 3, 8):
            rs = [mgpu.id_range(n, r, world) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(world - 1))
