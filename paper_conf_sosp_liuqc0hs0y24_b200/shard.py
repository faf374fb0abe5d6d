"""Multi-GPU plumbing for the batch `map`.

The batch map has no inter-iteration dependence (Table 1) and is the
outermost nest level (L180, L601), so ranks shard it: each rank owns a contiguous slice of
batch rows (batch-outermost layouts make every slice a contiguous memory slice), weights are
replicated, and nothing is exchanged during the forward.  The only collective is the optional
final gather of outputs to one rank (the north star's NCCL gather over NVLink), done with
torch.distributed (NCCL on GPUs, gloo in the CPU tests).  Pure plumbing: no arithmetic.
"""
from __future__ import annotations


def shard_rows(total: int, world: int, rank: int):
    """Contiguous [start, stop) of `total` batch rows for `rank` (sizes differ by at most 1)."""
    if world <= 0 or not (0 <= rank < world):
        raise ValueError("bad world/rank")
    base, extra = divmod(total, world)
    start = rank * base + min(rank, extra)
    stop = start + base + (1 if rank < extra else 0)
    return start, stop


def gather_rows(local, total_rows: int, dst: int = 0, group=None):
    """Gather every rank's batch slice (dim 0) to rank `dst`; returns the full tensor on `dst`
    and None elsewhere.  Uneven slices are padded to the largest slice for the collective."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    sizes = [shard_rows(total_rows, world, r) for r in range(world)]
    maxn = max(b - a for a, b in sizes)
    pad = torch.zeros((maxn,) + tuple(local.shape[1:]), dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    bufs = [torch.empty_like(pad) for _ in range(world)] if rank == dst else None
    dist.gather(pad, bufs, dst=dst, group=group)
    if rank != dst:
        return None
    return torch.cat([bufs[r][: b - a] for r, (a, b) in enumerate(sizes)], dim=0)
