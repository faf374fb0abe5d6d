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


class DevSlice:
    """A device address range that quacks like a tensor for ft.py's marshalling (`data_ptr()`):
    a peer rank's mapped output slice has no torch tensor of its own."""

    def __init__(self, ptr: int, shape, dtype):
        self.ptr, self.shape, self.dtype = ptr, tuple(shape), dtype

    def data_ptr(self):
        return self.ptr


def _elem_size(dtype):
    import torch
    return torch.empty((), dtype=dtype).element_size()


def _out_shapes(total_rows, seq, hidden, depth, dtype):
    import torch
    return {"y": ((total_rows, seq, hidden), dtype),
            "h_n": ((total_rows, depth, hidden), dtype),
            "c_n": ((total_rows, depth, hidden), torch.float32)}


class PeerGather:
    """NEXT-1: the output gather fused into the kernel's epilogue.

    Rank `dst` allocates the FULL output tensors (y [B_total][T][H], h_n / c_n [B_total][D][H])
    and exports them (ft_ipc_export); every other rank maps them into its OWN device's address
    space (ft_ipc_open: CUDA IPC with lazy peer access — on an NVSwitch node a peer-to-peer NVLink
    window) and passes ITS row slice as the `y` / `h_n` / `c_n` arguments of ft_stacked_lstm_fwd.
    The wavefront kernel's epilogue stores then land directly in rank `dst`'s HBM tile by tile,
    overlapping the transfer with the remaining diagonals — no gather launch, no staging copy.
    `done()` (stream sync + barrier) is the only synchronisation; after it rank `dst` owns the
    gathered outputs.  `close()` unmaps (collective).

    Batch rows are independent (the `map`, Table 1), so every rank writes a disjoint slice.
    Pure plumbing: allocation, handle exchange and slicing; the IPC calls are the library's own.
    Works across processes that share one GPU too (the 1-GPU tests).
    """

    def __init__(self, total_rows: int, seq: int, hidden: int, depth: int, dtype, device, dst: int = 0,
                 group=None):
        import torch
        import torch.distributed as dist
        from . import ft
        self.group = group
        self.dst = dst
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.total_rows = total_rows
        self.device = torch.device(device)
        self.shapes = _out_shapes(total_rows, seq, hidden, depth, dtype)
        self.full, self.opened = None, {}
        self.error = None  # set when this rank could not export / map the buffers (no exception:
                           # every rank still takes part in the collectives; see ok())
        handles = None
        if self.rank == dst:
            self.full = {k: torch.empty(shp, dtype=dt, device=self.device) for k, (shp, dt) in self.shapes.items()}
            handles = {}
            for k, v in self.full.items():
                st, h, off = ft.ft_ipc_export(v.data_ptr())
                if st != ft.FT_OK:
                    self.error = f"ft_ipc_export: {ft.ft_last_error()}"
                    handles = {"error": self.error}
                    break
                handles[k] = (h, off)
        obj = [handles]
        dist.broadcast_object_list(obj, src=dst, group=group)
        if self.rank != dst:
            if "error" in obj[0]:
                self.error = "root: " + obj[0]["error"]
            else:
                dev = self.device.index if self.device.index is not None else torch.cuda.current_device()
                for k, (h, off) in obj[0].items():
                    st, ptr = ft.ft_ipc_open(h, off, dev)
                    if st != ft.FT_OK:
                        self.error = f"ft_ipc_open: {ft.ft_last_error()}"
                        break
                    self.opened[k] = (ptr, off)

    def ok(self):
        """Collective: True when every rank mapped the buffers (else close() and fall back)."""
        import torch
        import torch.distributed as dist
        t = torch.tensor([0 if self.error else 1], dtype=torch.int32)
        if dist.get_backend(self.group) == "nccl":
            t = t.cuda()
        dist.all_reduce(t, op=dist.ReduceOp.MIN, group=self.group)
        return bool(t.item())

    def local(self):
        """This rank's row slice of the destination buffers (pass as `out=` to stacked_lstm)."""
        a, b = shard_rows(self.total_rows, self.world, self.rank)
        if self.rank == self.dst:
            return {k: v[a:b] for k, v in self.full.items()}
        out = {}
        for k, (shp, dt) in self.shapes.items():
            row_bytes = _elem_size(dt)
            for n in shp[1:]:
                row_bytes *= n
            out[k] = DevSlice(self.opened[k][0] + a * row_bytes, (b - a,) + tuple(shp[1:]), dt)
        return out

    def done(self):
        """Wait until every rank's kernel finished writing; then rank `dst` may read `full`."""
        import torch
        import torch.distributed as dist
        torch.cuda.synchronize()
        dist.barrier(group=self.group)
        return self.full if self.rank == self.dst else None

    def close(self):
        """Unmap the peer windows (collective: the root keeps its buffers until all closed)."""
        import torch.distributed as dist
        from . import ft
        for ptr, off in self.opened.values():
            ft.check(ft.ft_ipc_close(ptr, off))
        self.opened = {}
        dist.barrier(group=self.group)


class CommGather:
    """The north star's NCCL gather of y / h_n / c_n to rank `dst` through the library's own
    C-ABI (ft_comm_unique_id / ft_comm_init_rank / ft_comm_gather_rank), one process per GPU.
    The unique id travels over torch.distributed (control plane only).  Needs one distinct GPU
    per rank (NCCL refuses two ranks on one device)."""

    def __init__(self, total_rows: int, seq: int, hidden: int, depth: int, dtype, device, dst: int = 0,
                 group=None):
        import torch
        import torch.distributed as dist
        from . import ft
        self.dst = dst
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.total_rows = total_rows
        self.shapes = _out_shapes(total_rows, seq, hidden, depth, dtype)
        self.error, self.comm = None, None
        uid = None
        if self.rank == 0:
            st, uid = ft.ft_comm_unique_id()
            if st != ft.FT_OK:
                uid = None
        obj = [uid]
        dist.broadcast_object_list(obj, src=0, group=group)
        dev = torch.device(device)
        if obj[0] is None:
            self.error = "ft_comm_unique_id failed on rank 0"
        else:
            st, self.comm = ft.ft_comm_init_rank(self.world, self.rank, obj[0],
                                                 dev.index if dev.index is not None else torch.cuda.current_device())
            if st != ft.FT_OK:
                self.error = f"ft_comm_init_rank: {ft.ft_last_error()}"
                self.comm = None
        self.full = None
        if self.rank == dst:
            self.full = {k: torch.empty(shp, dtype=dt, device=dev) for k, (shp, dt) in self.shapes.items()}
        self.bytes = {}
        for k, (shp, dt) in self.shapes.items():
            row_bytes = _elem_size(dt)
            for n in shp[1:]:
                row_bytes *= n
            self.bytes[k] = [(b - a) * row_bytes for a, b in
                             (shard_rows(total_rows, self.world, r) for r in range(self.world))]

    def local(self):
        """Where this rank's forward writes: on the root its slice of the full buffers (the
        in-place root of the nccl.h gather convention), elsewhere fresh local tensors."""
        import torch
        a, b = shard_rows(self.total_rows, self.world, self.rank)
        if self.rank == self.dst:
            return {k: v[a:b] for k, v in self.full.items()}
        dev = torch.device("cuda", torch.cuda.current_device())
        return {k: torch.empty((b - a,) + tuple(shp[1:]), dtype=dt, device=dev)
                for k, (shp, dt) in self.shapes.items()}

    def ok(self):
        """Collective: True when every rank has a communicator."""
        import torch
        import torch.distributed as dist
        t = torch.tensor([0 if self.error else 1], dtype=torch.int32)
        if dist.get_backend() == "nccl":
            t = t.cuda()
        dist.all_reduce(t, op=dist.ReduceOp.MIN)
        return bool(t.item())

    def gather(self, outs, stream_ptr):
        from . import ft
        for k in ("y", "h_n", "c_n"):
            recv = self.full[k].data_ptr() if self.full is not None else None
            ft.check(ft.ft_comm_gather_rank(self.comm, outs[k].data_ptr(), recv, self.bytes[k], self.dst,
                                            stream_ptr))

    def close(self):
        from . import ft
        if self.comm:
            ft.check(ft.ft_comm_destroy(self.comm))
            self.comm = None
