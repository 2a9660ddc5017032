"""Multi-GPU collage plumbing.  Two partitions:

* by image: query blocks are split into contiguous row-major ranges, one per
  rank (blocks are independent), and the per-block winners are
  collected on rank 0 with one gather;
* by bucket (AP_SCHED_TABLE): the L * B (block, table) units, in (table,
  bucket) order, are split into contiguous ranges, so each LSH bucket -- and
  the records it lists -- is read by one rank; a block's units may land on
  several ranks, so the winners are combined with one MIN reduction of the
  64-bit (dist << 32 | idx) words (R-A3's lexicographic order).

* by records (AP_SCHED_TABLE with ap_collage_in.id_begin/id_end): rank r
  runs every unit but reads only candidates whose record id lies in its
  contiguous slice of the file, so each GPU's page cache holds one shard of
  the file and every record is filled by exactly one rank (a data-parallel
  split of the file itself); winners are MIN-reduced like the bucket split.

Two ways to combine the winners:

* fused (SharedWinners, the default): rank 0's winners array is mapped into
  every rank's process with CUDA IPC (ap_ipc_export / ap_ipc_import) and each
  rank's collage kernel folds its blocks' results straight into it with a
  system-scope 64-bit atomic min over NVLink (ap_collage_in.flags =
  AP_COLLAGE_ACCUMULATE | AP_COLLAGE_SYSTEM): no collective in the data path,
  the combine overlaps the other ranks' kernels.  The arithmetic is in the
  kernel; this module only exchanges the IPC handle and synchronises.
* NCCL (gather_winners / reduce_winners_min): one gather or one MIN reduce
  over torch.distributed, the baseline the fused path replaces.

gloo in the CPU tests.  Marshalling only.
"""


def block_range(nblocks, rank, world):
    """Contiguous range [b0, b1) of rank `rank` (sizes differ by at most 1)."""
    return rank * nblocks // world, (rank + 1) * nblocks // world


def gather_winners(win, rank, world, dist, nblocks, dst=0):
    """Gather every rank's winners (int32 [b1-b0, 2]) to `dst`; returns the
    full [nblocks, 2] tensor on dst, None elsewhere.  Ranges may differ by
    one block, so each rank pads to the largest range before the gather."""
    import torch
    if world == 1:
        return win
    rows = -(-nblocks // world)
    # gloo gathers host tensors; NCCL gathers device tensors over NVLink
    dev = win.device if dist.get_backend() == "nccl" else "cpu"
    pad = torch.full((rows, 2), -1, dtype=win.dtype, device=dev)
    pad[:win.shape[0]] = win.to(dev)
    bufs = [torch.empty_like(pad) for _ in range(world)] if rank == dst else None
    dist.gather(pad, bufs, dst=dst)
    if rank != dst:
        return None
    parts = []
    for r in range(world):
        b0, b1 = block_range(nblocks, r, world)
        parts.append(bufs[r][:b1 - b0])
    return torch.cat(parts)


def unit_range(nunits, rank, world):
    """Contiguous range [u0, u1) of the sorted units for rank `rank`."""
    return rank * nunits // world, (rank + 1) * nunits // world


def id_range(nrecords, rank, world):
    """Contiguous record-id slice [i0, i1) of rank `rank` (by-records split)."""
    return rank * nrecords // world, (rank + 1) * nrecords // world


def reduce_winners_min(win, rank, world, dist, dst=0):
    """Combine per-rank partial winners (int32 [B, 2] = (idx, dist) words, the
    empty sentinel 0xFFFFFFFF where a rank saw no candidate) into the
    lexicographic (dist, idx) minimum on `dst`; returns it there, None
    elsewhere.  The pair read as one little-endian u64 is dist << 32 | idx;
    flipping its sign bit maps unsigned order onto int64 order, so one
    signed MIN reduction does it."""
    import torch
    if world == 1:
        return win
    dev = win.device if dist.get_backend() == "nccl" else "cpu"
    flip = torch.tensor(-(1 << 63), dtype=torch.int64, device=dev)
    w64 = win.to(dev).contiguous().view(torch.int64).view(-1) ^ flip
    dist.reduce(w64, dst=dst, op=dist.ReduceOp.MIN)
    if rank != dst:
        return None
    return (w64 ^ flip).view(torch.int32).view(-1, 2)


class SharedWinners:
    """Rank 0's winners array, addressable by every rank's kernels (CUDA IPC).

    `ptr(b0)` is the device address a rank passes to ap_collage_run as
    winners_dev (with flags AP_COLLAGE_ACCUMULATE | AP_COLLAGE_SYSTEM) for
    its partition starting at block b0.  Per step: `begin(stream)` on every
    rank (rank 0 sets the sentinels, all ranks wait for it), the ranks' kernels
    accumulate, `end()` on every rank; then rank 0's `result` holds the
    combined winners."""

    def __init__(self, ap, nblocks, rank, world, dist, device):
        import torch
        self.ap, self.rank, self.world, self.dist = ap, rank, world, dist
        self.nblocks = nblocks
        self.result = None
        self._mapped = None
        if rank == 0:
            self.result = torch.empty((nblocks, 2), dtype=torch.int32, device=device)
            blob = [bytes(ap.ap_ipc_export(self.result))] if world > 1 else [None]
        else:
            blob = [None]
        if world > 1:
            dist.broadcast_object_list(blob, src=0)
        if rank == 0:
            self._base = self.result.data_ptr()
        else:
            h = ap.ap_ipc_handle_t.from_buffer_copy(blob[0])
            self._mapped = ap.ap_ipc_import(h, device.index if device.index is not None else 0)
            self._base = self._mapped

    def ptr(self, b0=0):
        return self._base + 8 * b0

    def begin(self, stream=None):
        import torch
        if self.rank == 0:
            self.ap.ap_winners_init(self.result, self.nblocks, stream)
            torch.cuda.synchronize()
        if self.world > 1:
            self.dist.barrier()

    def end(self):
        import torch
        torch.cuda.synchronize()
        if self.world > 1:
            self.dist.barrier()

    def close(self):
        if self._mapped is not None:
            self.ap.ap_ipc_close(self._mapped)
            self._mapped = None
