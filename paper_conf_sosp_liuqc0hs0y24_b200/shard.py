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


class PeerGather:
    """NEXT-1: the output gather fused into the kernel's epilogue.

    Rank `dst` allocates the FULL output tensors (y [B_total][T][H], h_n / c_n [B_total][D][H]);
    every rank maps them into its own address space (CUDA IPC; on an NVSwitch node the mapping is
    a peer-to-peer NVLink window) and passes ITS row slice of rank `dst`'s buffers as the `y` /
    `h_n` / `c_n` arguments of ft_stacked_lstm_fwd.  The wavefront kernel's epilogue stores then
    land directly in rank `dst`'s HBM tile by tile, overlapping the transfer with the remaining
    diagonals — no separate gather launch, no staging copy.  `done()` (stream sync + barrier) is
    the only synchronisation; after it rank `dst` owns the gathered outputs.

    Batch rows are independent (the `map`, Table 1), so every rank writes a disjoint slice.
    Pure plumbing: buffer allocation, handle exchange and slicing.  Requires CUDA tensors and
    ranks on one node; works across processes that share a GPU too (used by the 1-GPU test).
    """

    def __init__(self, total_rows: int, seq: int, hidden: int, depth: int, dtype, device, dst: int = 0,
                 group=None):
        import torch
        import torch.distributed as dist
        from torch.multiprocessing.reductions import reduce_tensor
        self.group = group
        self.dst = dst
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.total_rows = total_rows
        if self.rank == dst:
            full = {"y": torch.empty((total_rows, seq, hidden), dtype=dtype, device=device),
                    "h_n": torch.empty((total_rows, depth, hidden), dtype=dtype, device=device),
                    "c_n": torch.empty((total_rows, depth, hidden), dtype=torch.float32, device=device)}
            handles = {k: reduce_tensor(v) for k, v in full.items()}
        else:
            full, handles = None, None
        obj = [handles]
        dist.broadcast_object_list(obj, src=dst, group=group)
        if self.rank != dst:
            full = {k: fn(*args) for k, (fn, args) in obj[0].items()}
        self.full = full

    def local(self):
        """This rank's row slice of the destination buffers (pass as `out=` to stacked_lstm)."""
        a, b = shard_rows(self.total_rows, self.world, self.rank)
        return {k: v[a:b] for k, v in self.full.items()}

    def done(self):
        """Wait until every rank's kernel finished writing; then rank `dst` may read `full`."""
        import torch
        import torch.distributed as dist
        torch.cuda.synchronize()
        dist.barrier(group=self.group)
        return self.full if self.rank == self.dst else None
