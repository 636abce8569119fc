"""Multi-GPU partitioning of a frame batch.

Frames are independent units (each has its own pEdge mean), so a
batch is split into contiguous frame ranges, one per rank (one process per
GPU), with no collective on the data path.  torch.distributed is used only for
the plumbing: a barrier and the max-over-ranks of the measured times.
"""


def frame_range(n, world, rank):
    """Contiguous [start, start+count) of n frames for `rank` of `world`
    (the first n % world ranks get one extra frame)."""
    if world < 1 or not 0 <= rank < world or n < 0:
        raise ValueError("bad partition request")
    base, rem = divmod(n, world)
    start = rank * base + min(rank, rem)
    return start, base + (1 if rank < rem else 0)


def max_over_ranks(x, device=None):
    """Max of a float over all ranks of the default process group (identity
    when torch.distributed is not initialised)."""
    import torch
    import torch.distributed as dist

    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def barrier():
    import torch.distributed as dist

    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.barrier()
