"""Multi-GPU collage plumbing: query blocks are split
into contiguous row-major ranges, one per rank (blocks are independent,
PAPER.md:419), and the per-block winners are collected on rank 0 with one
gather (NCCL over NVLink on GPUs; gloo in the CPU tests).  Marshalling only.
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
