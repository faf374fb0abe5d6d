"""Thin ctypes binding of libft.so (include/ft.h).  Argument marshalling only.

Two layers:
  * the raw C-ABI names (`ft_stacked_lstm_fwd`, `ft_dilated_rnn_fwd`, `ft_grid_rnn_fwd`, the
    `*_workspace_size` queries, `ft_wavefront_cells`, ...) taking ints / raw pointers exactly
    as the header declares them;
  * torch-tensor conveniences (`stacked_lstm`, `dilated_rnn`, `grid_rnn`) that allocate the
    outputs and the workspace with torch (PyTorch is plumbing: device memory and streams) and
    call the raw entry point.  Every step of the computation runs in the library's kernels.

There is no fallback: if libft.so is missing or a call fails, an exception is raised.
"""
from __future__ import annotations

import ctypes
import os

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("FT_LIB_PATH") or os.path.join(PKG, "libft.so")  # override: A/B timing of two builds

FT_OK, FT_ERR_INVALID_ARGUMENT, FT_ERR_UNSUPPORTED, FT_ERR_CUDA, FT_ERR_NCCL = 0, 1, 2, 3, 4
FT_ERR_WORKSPACE_TOO_SMALL = 5
FT_F32, FT_BF16 = 0, 1
FT_MAX_DEPTH = 64

# every symbol include/ft.h declares (checked by tests/test_abi.py against the header)
EXPORTS = (
    "ft_version", "ft_status_string", "ft_last_error", "ft_last_launch", "ft_set_l2_persist",
    "ft_stacked_lstm_workspace_size", "ft_stacked_lstm_fwd",
    "ft_stacked_lstm_hostio_workspace_size", "ft_stacked_lstm_fwd_hostio",
    "ft_stacked_rnn_workspace_size", "ft_stacked_rnn_fwd",
    "ft_stacked_lstm_layerwise_workspace_size", "ft_stacked_lstm_layerwise_fwd",
    "ft_b2b_gemm_fwd",
    "ft_dilated_rnn_workspace_size", "ft_dilated_rnn_fwd",
    "ft_grid_rnn_workspace_size", "ft_grid_rnn_fwd",
    "ft_wavefront_cells", "ft_wavefront_cells_banded", "ft_tile_walk", "ft_ssa_slots",
    "ft_comm_create", "ft_comm_gather", "ft_comm_destroy",
    "ft_comm_unique_id", "ft_comm_init_rank", "ft_comm_gather_rank",
    "ft_ipc_export", "ft_ipc_open", "ft_ipc_close",
)
FT_COMM_ID_BYTES = 128
FT_IPC_HANDLE_BYTES = 64


class FTError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{status_string(status)}: {msg}")
        self.status = status


_lib = None
_c_int, _c_size, _c_vp, _c_ll = ctypes.c_int, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_longlong


def lib():
    """Load libft.so (in-tree).  Raises if it was not built — no CPU or library fallback."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run `python -m paper_conf_sosp_liuqc0hs0y24_b200.build`")
        L = ctypes.CDLL(LIB_PATH)
        if os.environ.get("FT_LIB_PATH"):  # A/B timing of an older build: tolerate missing symbols
            class _Tolerant:
                def __init__(self, lib):
                    object.__setattr__(self, "_l", lib)

                def __getattr__(self, name):
                    try:
                        return getattr(self._l, name)
                    except AttributeError:
                        return _Dummy()

                def __setattr__(self, name, value):
                    setattr(self._l, name, value)

            class _Dummy:
                restype = None
                argtypes = None

                def __call__(self, *a):
                    raise AttributeError("symbol missing in this build")
            L = _Tolerant(L)
        L.ft_version.restype = _c_int
        L.ft_set_l2_persist.restype = _c_int
        L.ft_set_l2_persist.argtypes = [_c_int]
        L.ft_status_string.restype = ctypes.c_char_p
        L.ft_status_string.argtypes = [_c_int]
        L.ft_last_error.restype = ctypes.c_char_p
        L.ft_last_launch.restype = ctypes.c_char_p
        L.ft_stacked_lstm_workspace_size.restype = _c_size
        L.ft_stacked_lstm_workspace_size.argtypes = [_c_int] * 6
        L.ft_dilated_rnn_workspace_size.restype = _c_size
        L.ft_dilated_rnn_workspace_size.argtypes = [_c_int, _c_int, _c_int, _c_int, _c_vp, _c_int, _c_int]
        L.ft_grid_rnn_workspace_size.restype = _c_size
        L.ft_grid_rnn_workspace_size.argtypes = [_c_int] * 7
        L.ft_stacked_lstm_fwd.restype = _c_int
        L.ft_stacked_lstm_fwd.argtypes = [_c_int] * 5 + [_c_vp] * 9 + [_c_vp, _c_size, _c_vp]
        L.ft_dilated_rnn_fwd.restype = _c_int
        L.ft_dilated_rnn_fwd.argtypes = [_c_int] * 4 + [_c_vp, _c_int] + [_c_vp] * 9 + [_c_vp, _c_size, _c_vp]
        L.ft_grid_rnn_fwd.restype = _c_int
        L.ft_grid_rnn_fwd.argtypes = [_c_int] * 6 + [_c_vp] * 10 + [_c_vp, _c_size, _c_vp]
        L.ft_stacked_lstm_hostio_workspace_size.restype = _c_size
        L.ft_stacked_lstm_hostio_workspace_size.argtypes = [_c_int] * 5
        L.ft_stacked_lstm_fwd_hostio.restype = _c_int
        L.ft_stacked_lstm_fwd_hostio.argtypes = [_c_int] * 5 + [_c_vp] * 7 + [_c_vp, _c_size, _c_vp]
        L.ft_stacked_rnn_workspace_size.restype = _c_size
        L.ft_stacked_rnn_workspace_size.argtypes = [_c_int] * 5
        L.ft_stacked_rnn_fwd.restype = _c_int
        L.ft_stacked_rnn_fwd.argtypes = [_c_int] * 5 + [_c_vp] * 3 + [_c_vp, _c_size, _c_vp]
        L.ft_stacked_lstm_layerwise_workspace_size.restype = _c_size
        L.ft_stacked_lstm_layerwise_workspace_size.argtypes = [_c_int] * 5
        L.ft_stacked_lstm_layerwise_fwd.restype = _c_int
        L.ft_stacked_lstm_layerwise_fwd.argtypes = [_c_int] * 5 + [_c_vp] * 9 + [_c_vp, _c_size, _c_vp]
        L.ft_b2b_gemm_fwd.restype = _c_int
        L.ft_b2b_gemm_fwd.argtypes = [_c_int] * 5 + [_c_vp] * 4 + [_c_vp]
        L.ft_comm_create.restype = _c_int
        L.ft_comm_create.argtypes = [_c_int, _c_vp, ctypes.POINTER(_c_vp)]
        L.ft_comm_gather.restype = _c_int
        L.ft_comm_gather.argtypes = [_c_vp, _c_vp, _c_vp, _c_vp, _c_int, _c_vp]
        L.ft_comm_destroy.restype = _c_int
        L.ft_comm_destroy.argtypes = [_c_vp]
        L.ft_comm_unique_id.restype = _c_int
        L.ft_comm_unique_id.argtypes = [_c_vp]
        L.ft_comm_init_rank.restype = _c_int
        L.ft_comm_init_rank.argtypes = [_c_int, _c_int, _c_vp, _c_int, ctypes.POINTER(_c_vp)]
        L.ft_comm_gather_rank.restype = _c_int
        L.ft_comm_gather_rank.argtypes = [_c_vp, _c_vp, _c_vp, _c_vp, _c_int, _c_vp]
        L.ft_ipc_export.restype = _c_int
        L.ft_ipc_export.argtypes = [_c_vp, _c_vp, ctypes.POINTER(_c_size)]
        L.ft_ipc_open.restype = _c_int
        L.ft_ipc_open.argtypes = [_c_vp, _c_size, _c_int, ctypes.POINTER(_c_vp)]
        L.ft_ipc_close.restype = _c_int
        L.ft_ipc_close.argtypes = [_c_vp, _c_size]
        L.ft_wavefront_cells.restype = _c_ll
        L.ft_wavefront_cells.argtypes = [_c_int] * 4 + [_c_vp, _c_ll]
        L.ft_wavefront_cells_banded.restype = _c_ll
        L.ft_wavefront_cells_banded.argtypes = [_c_int] * 6 + [_c_vp, _c_ll]
        L.ft_tile_walk.restype = _c_ll
        L.ft_ssa_slots.restype = _c_ll
        L.ft_ssa_slots.argtypes = [_c_int, _c_int, _c_vp, _c_int, _c_vp, _c_vp]
        L.ft_tile_walk.argtypes = [_c_int] * 8 + [_c_vp, _c_ll]
        _lib = L
    return _lib


# ------------------------------------------------------------------------------ raw C ABI
def ft_version() -> int:
    return lib().ft_version()


def ft_set_l2_persist(mib: int) -> int:
    """Persisting-L2 window size for streaming calls (-1 auto, 0 off, else MiB); returns a status."""
    return lib().ft_set_l2_persist(mib)


def status_string(s: int) -> str:
    return lib().ft_status_string(s).decode()


def ft_last_error() -> str:
    return lib().ft_last_error().decode()


def ft_last_launch() -> str:
    """Launch configuration and schedule of the last forward on this thread (diagnostic)."""
    return lib().ft_last_launch().decode()


def ft_stacked_lstm_workspace_size(batch, seq, hidden, depth, dt, h_all_provided):
    return lib().ft_stacked_lstm_workspace_size(batch, seq, hidden, depth, dt, int(h_all_provided))


def _int_array(vals):
    arr = (ctypes.c_int * len(vals))(*[int(v) for v in vals])
    return arr


def ft_dilated_rnn_workspace_size(batch, seq, hidden, depth, dilations, dt, h_all_provided):
    arr = _int_array(dilations) if dilations is not None else None
    return lib().ft_dilated_rnn_workspace_size(batch, seq, hidden, depth,
                                               ctypes.cast(arr, _c_vp) if arr is not None else None,
                                               dt, int(h_all_provided))


def ft_grid_rnn_workspace_size(batch, len_x, len_y, hidden, depth, dt, h_all_provided):
    return lib().ft_grid_rnn_workspace_size(batch, len_x, len_y, hidden, depth, dt, int(h_all_provided))


def ft_stacked_lstm_fwd(batch, seq, hidden, depth, dt, x, W, U, b, y, h_n, c_n, h_all, c_all,
                        workspace, workspace_bytes, stream) -> int:
    return lib().ft_stacked_lstm_fwd(batch, seq, hidden, depth, dt, x, W, U, b, y, h_n, c_n,
                                     h_all, c_all, workspace, workspace_bytes, stream)


def ft_stacked_lstm_hostio_workspace_size(batch, seq, hidden, depth, dt):
    return lib().ft_stacked_lstm_hostio_workspace_size(batch, seq, hidden, depth, dt)


def ft_stacked_lstm_fwd_hostio(batch, seq, hidden, depth, dt, x_host, W, U, b, y_host, h_n_host,
                               c_n_host, workspace, workspace_bytes, stream) -> int:
    return lib().ft_stacked_lstm_fwd_hostio(batch, seq, hidden, depth, dt, x_host, W, U, b,
                                            y_host, h_n_host, c_n_host, workspace,
                                            workspace_bytes, stream)


def ft_stacked_rnn_workspace_size(batch, seq, hidden, depth, dt):
    return lib().ft_stacked_rnn_workspace_size(batch, seq, hidden, depth, dt)


def ft_stacked_rnn_fwd(batch, seq, hidden, depth, dt, x, W, ys, workspace, workspace_bytes,
                       stream) -> int:
    return lib().ft_stacked_rnn_fwd(batch, seq, hidden, depth, dt, x, W, ys, workspace,
                                    workspace_bytes, stream)


def ft_stacked_lstm_layerwise_workspace_size(batch, seq, hidden, depth, dt):
    return lib().ft_stacked_lstm_layerwise_workspace_size(batch, seq, hidden, depth, dt)


def ft_stacked_lstm_layerwise_fwd(batch, seq, hidden, depth, dt, x, W, U, b, y, h_n, c_n, h_all,
                                  c_all, workspace, workspace_bytes, stream) -> int:
    return lib().ft_stacked_lstm_layerwise_fwd(batch, seq, hidden, depth, dt, x, W, U, b, y, h_n,
                                               c_n, h_all, c_all, workspace, workspace_bytes, stream)


def ft_b2b_gemm_fwd(M, N, K, P, dt, A, B, C, D, stream) -> int:
    return lib().ft_b2b_gemm_fwd(M, N, K, P, dt, A, B, C, D, stream)


def ft_dilated_rnn_fwd(batch, seq, hidden, depth, dilations, dt, x, W, U, b, y, h_n, c_n, h_all,
                       c_all, workspace, workspace_bytes, stream) -> int:
    arr = _int_array(dilations) if dilations is not None else None
    return lib().ft_dilated_rnn_fwd(batch, seq, hidden, depth,
                                    ctypes.cast(arr, _c_vp) if arr is not None else None, dt,
                                    x, W, U, b, y, h_n, c_n, h_all, c_all, workspace,
                                    workspace_bytes, stream)


def ft_grid_rnn_fwd(batch, len_x, len_y, hidden, depth, dt, x, ys, W, U, b, out, h_n, c_n,
                    h_all, c_all, workspace, workspace_bytes, stream) -> int:
    return lib().ft_grid_rnn_fwd(batch, len_x, len_y, hidden, depth, dt, x, ys, W, U, b, out,
                                 h_n, c_n, h_all, c_all, workspace, workspace_bytes, stream)


def ft_wavefront_cells(kind, depth, len_a, len_b=1):
    """Wavefront cell order as a list of (diagonal, d, i, j) — host only."""
    n = lib().ft_wavefront_cells(kind, depth, len_a, len_b, None, 0)
    if n < 0:
        raise FTError(FT_ERR_INVALID_ARGUMENT, "bad schedule query")
    buf = (ctypes.c_int * (4 * n))()
    lib().ft_wavefront_cells(kind, depth, len_a, len_b, ctypes.cast(buf, _c_vp), n)
    return [tuple(buf[4 * k:4 * k + 4]) for k in range(n)]


def ft_wavefront_cells_banded(kind, depth, len_a, len_b=1, band=0, skew=1):
    """Cell order of the layer-banded wavefront (kind 0): list of (diagonal, d, i, j) — host only."""
    n = lib().ft_wavefront_cells_banded(kind, depth, len_a, len_b, band, skew, None, 0)
    if n < 0:
        raise FTError(FT_ERR_INVALID_ARGUMENT, "bad schedule query")
    buf = (ctypes.c_int * (4 * n))()
    lib().ft_wavefront_cells_banded(kind, depth, len_a, len_b, band, skew, ctypes.cast(buf, _c_vp), n)
    return [tuple(buf[4 * k:4 * k + 4]) for k in range(n)]


def ft_tile_walk(depth, seq, band, skew, owner, ntiles_n, worker, nworkers):
    """One worker's tile sequence [(d, t, n), ...] of the bf16 kernel's walk — host only."""
    n = lib().ft_tile_walk(depth, seq, band, skew, owner, ntiles_n, worker, nworkers, None, 0)
    if n < 0:
        raise FTError(FT_ERR_INVALID_ARGUMENT, "bad tile-walk query")
    buf = (ctypes.c_int * (3 * max(n, 1)))()
    lib().ft_tile_walk(depth, seq, band, skew, owner, ntiles_n, worker, nworkers, ctypes.cast(buf, _c_vp), n)
    return [tuple(buf[3 * k:3 * k + 3]) for k in range(n)]


def ft_ssa_slots(depth, seq, dilations, band):
    """(rows, off[], mask[]) of the streaming kernel's SSA ring layout — host only."""
    dil = _int_array(dilations)
    off = (ctypes.c_int * depth)()
    mask = (ctypes.c_int * depth)()
    rows = lib().ft_ssa_slots(depth, seq, ctypes.cast(dil, _c_vp), band, ctypes.cast(off, _c_vp),
                              ctypes.cast(mask, _c_vp))
    if rows < 0:
        raise FTError(FT_ERR_INVALID_ARGUMENT, "bad ssa-slot query")
    return rows, list(off), list(mask)


def ft_comm_create(devices):
    """Returns (status, comm handle) for an NCCL communicator over `devices` (one process)."""
    arr = _int_array(devices)
    out = _c_vp()
    st = lib().ft_comm_create(len(devices), ctypes.cast(arr, _c_vp), ctypes.byref(out))
    return st, out.value


def ft_comm_gather(comm, send_ptrs, recv_ptr, nbytes, root, stream_ptrs):
    n = len(send_ptrs)
    send = (_c_vp * n)(*send_ptrs)
    sizes = (_c_size * n)(*nbytes)
    streams = (_c_vp * n)(*stream_ptrs)
    return lib().ft_comm_gather(comm, ctypes.cast(send, _c_vp), recv_ptr, ctypes.cast(sizes, _c_vp),
                                root, ctypes.cast(streams, _c_vp))


def ft_comm_destroy(comm):
    return lib().ft_comm_destroy(comm)


def ft_comm_unique_id():
    """Returns (status, bytes) — the opaque FT_COMM_ID_BYTES id one rank ships to the others."""
    buf = ctypes.create_string_buffer(FT_COMM_ID_BYTES)
    st = lib().ft_comm_unique_id(ctypes.cast(buf, _c_vp))
    return st, buf.raw


def ft_comm_init_rank(nranks, rank, uid, device):
    """Returns (status, comm handle) — this process's rank of an NCCL communicator."""
    buf = ctypes.create_string_buffer(bytes(uid), FT_COMM_ID_BYTES)
    out = _c_vp()
    st = lib().ft_comm_init_rank(nranks, rank, ctypes.cast(buf, _c_vp), device, ctypes.byref(out))
    return st, out.value


def ft_comm_gather_rank(comm, send_ptr, recv_ptr, nbytes, root, stream_ptr):
    sizes = (_c_size * len(nbytes))(*nbytes)
    return lib().ft_comm_gather_rank(comm, send_ptr, recv_ptr, ctypes.cast(sizes, _c_vp), root, stream_ptr)


def ft_ipc_export(dev_ptr):
    """Returns (status, handle bytes, offset) of the allocation holding `dev_ptr`."""
    buf = ctypes.create_string_buffer(FT_IPC_HANDLE_BYTES)
    off = _c_size()
    st = lib().ft_ipc_export(dev_ptr, ctypes.cast(buf, _c_vp), ctypes.byref(off))
    return st, buf.raw, off.value


def ft_ipc_open(handle, offset, device):
    """Returns (status, device pointer) of an exported allocation mapped into `device`."""
    buf = ctypes.create_string_buffer(bytes(handle), FT_IPC_HANDLE_BYTES)
    out = _c_vp()
    st = lib().ft_ipc_open(ctypes.cast(buf, _c_vp), offset, device, ctypes.byref(out))
    return st, out.value


def ft_ipc_close(dev_ptr, offset):
    return lib().ft_ipc_close(dev_ptr, offset)


def check(status: int):
    if status != FT_OK:
        raise FTError(status, ft_last_error())


# ------------------------------------------------------------------------------ torch helpers
def _torch():
    import torch
    return torch


def _dt(t):
    torch = _torch()
    if t.dtype == torch.bfloat16:
        return FT_BF16
    if t.dtype == torch.float32:
        return FT_F32
    raise TypeError(f"unsupported dtype {t.dtype}")


def _ptr(t):
    return None if t is None else t.data_ptr()


def _stream_ptr(stream):
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream


class Workspace:
    """A reusable device workspace (torch uint8 buffer) grown on demand."""

    def __init__(self, device=None):
        self.buf = None
        self.device = device

    def get(self, nbytes, device):
        torch = _torch()
        if self.buf is None or self.buf.numel() < nbytes or self.buf.device != device:
            self.buf = torch.empty(max(nbytes, 256), dtype=torch.uint8, device=device)
        return self.buf


def stacked_lstm(x, W, U, b, want_all=False, dilations=None, stream=None, workspace=None, out=None):
    """Stacked (or, with `dilations`, dilated) LSTM forward on the GPU through the C ABI.

    x [B][T][H] (bf16 or fp32 CUDA tensor), W/U [D][4][H][H] (same dtype), b [D][4][H] fp32.
    Returns dict y, h_n, c_n (+ h_all, c_all when want_all)."""
    torch = _torch()
    B, T, H = x.shape
    D = W.shape[0]
    dt = _dt(x)
    dev = x.device
    o = out or {}
    y = o.get("y") if o.get("y") is not None else torch.empty((B, T, H), dtype=x.dtype, device=dev)
    h_n = o.get("h_n") if o.get("h_n") is not None else torch.empty((B, D, H), dtype=x.dtype, device=dev)
    c_n = o.get("c_n") if o.get("c_n") is not None else torch.empty((B, D, H), dtype=torch.float32, device=dev)
    h_all = torch.empty((B, D, T, H), dtype=x.dtype, device=dev) if want_all else None
    c_all = torch.empty((B, D, T, H), dtype=torch.float32, device=dev) if want_all else None
    if dilations is None:
        nbytes = ft_stacked_lstm_workspace_size(B, T, H, D, dt, h_all is not None)
    else:
        nbytes = ft_dilated_rnn_workspace_size(B, T, H, D, dilations, dt, h_all is not None)
    ws = (workspace or Workspace()).get(nbytes, dev)
    sp = _stream_ptr(stream)
    if dilations is None:
        st = ft_stacked_lstm_fwd(B, T, H, D, dt, _ptr(x), _ptr(W), _ptr(U), _ptr(b), _ptr(y),
                                 _ptr(h_n), _ptr(c_n), _ptr(h_all), _ptr(c_all), ws.data_ptr(),
                                 ws.numel(), sp)
    else:
        st = ft_dilated_rnn_fwd(B, T, H, D, dilations, dt, _ptr(x), _ptr(W), _ptr(U), _ptr(b),
                                _ptr(y), _ptr(h_n), _ptr(c_n), _ptr(h_all), _ptr(c_all),
                                ws.data_ptr(), ws.numel(), sp)
    check(st)
    r = dict(y=y, h_n=h_n, c_n=c_n)
    if want_all:
        r.update(h_all=h_all, c_all=c_all)
    return r


def stacked_lstm_layerwise(x, W, U, b, want_all=False, stream=None, workspace=None):
    """The layer-sequential comparison schedule (NEXT-2): same inputs and outputs as
    `stacked_lstm` (bf16 only), computed one layer after another with a hoisted input GEMM."""
    torch = _torch()
    B, T, H = x.shape
    D = W.shape[0]
    dt = _dt(x)
    dev = x.device
    y = torch.empty((B, T, H), dtype=x.dtype, device=dev)
    h_n = torch.empty((B, D, H), dtype=x.dtype, device=dev)
    c_n = torch.empty((B, D, H), dtype=torch.float32, device=dev)
    h_all = torch.empty((B, D, T, H), dtype=x.dtype, device=dev) if want_all else None
    c_all = torch.empty((B, D, T, H), dtype=torch.float32, device=dev) if want_all else None
    nbytes = ft_stacked_lstm_layerwise_workspace_size(B, T, H, D, dt)
    ws = (workspace or Workspace()).get(nbytes, dev)
    check(ft_stacked_lstm_layerwise_fwd(B, T, H, D, dt, _ptr(x), _ptr(W), _ptr(U), _ptr(b), _ptr(y),
                                        _ptr(h_n), _ptr(c_n), _ptr(h_all), _ptr(c_all),
                                        ws.data_ptr(), ws.numel(), _stream_ptr(stream)))
    r = dict(y=y, h_n=h_n, c_n=c_n)
    if want_all:
        r.update(h_all=h_all, c_all=c_all)
    return r


def dilated_rnn(x, W, U, b, dilations, **kw):
    return stacked_lstm(x, W, U, b, dilations=list(dilations), **kw)


def grid_rnn(x, ys, W, U, b, want_all=False, stream=None, workspace=None):
    """Grid LSTM forward.  x [B][Lx][H], ys [B][Ly][H], W [D][2][4][H][H], U [D][2][4][2H][H],
    b [D][2][4][H] fp32.  Returns dict out [B][Lx][Ly][2][H], h_n, c_n (+ h_all, c_all)."""
    torch = _torch()
    B, Lx, H = x.shape
    Ly = ys.shape[1]
    D = W.shape[0]
    dt = _dt(x)
    dev = x.device
    out = torch.empty((B, Lx, Ly, 2, H), dtype=x.dtype, device=dev)
    h_n = torch.empty((B, D, 2, H), dtype=x.dtype, device=dev)
    c_n = torch.empty((B, D, 2, H), dtype=torch.float32, device=dev)
    h_all = torch.empty((B, D, Lx, Ly, 2, H), dtype=x.dtype, device=dev) if want_all else None
    c_all = torch.empty((B, D, Lx, Ly, 2, H), dtype=torch.float32, device=dev) if want_all else None
    nbytes = ft_grid_rnn_workspace_size(B, Lx, Ly, H, D, dt, h_all is not None)
    ws = (workspace or Workspace()).get(nbytes, dev)
    st = ft_grid_rnn_fwd(B, Lx, Ly, H, D, dt, _ptr(x), _ptr(ys), _ptr(W), _ptr(U), _ptr(b),
                         _ptr(out), _ptr(h_n), _ptr(c_n), _ptr(h_all), _ptr(c_all),
                         ws.data_ptr(), ws.numel(), _stream_ptr(stream))
    check(st)
    r = dict(out=out, h_n=h_n, c_n=c_n)
    if want_all:
        r.update(h_all=h_all, c_all=c_all)
    return r


def stacked_rnn(x, W, stream=None, workspace=None):
    """Listing 1's stacked linear RNN (y = x@w + s) through the C ABI.
    x [B][T][H] (bf16 / fp32 CUDA), W [D][H][H] → ys [B][D][T][H] (every layer's output)."""
    torch = _torch()
    B, T, H = x.shape
    D = W.shape[0]
    dt = _dt(x)
    ys = torch.empty((B, D, T, H), dtype=x.dtype, device=x.device)
    nbytes = ft_stacked_rnn_workspace_size(B, T, H, D, dt)
    ws = (workspace or Workspace()).get(nbytes, x.device)
    check(ft_stacked_rnn_fwd(B, T, H, D, dt, _ptr(x), _ptr(W), _ptr(ys), ws.data_ptr(), ws.numel(),
                             _stream_ptr(stream)))
    return ys


def b2b_gemm(A, B, C, stream=None):
    """Back-to-back GEMMs (Table 6): D = (A @ B) @ C, one fused tcgen05 kernel.
    A [M][64], B [64][N], C [N][64] bf16 CUDA tensors → D [M][64] fp32."""
    torch = _torch()
    M, K = A.shape
    N = B.shape[1]
    P = C.shape[1]
    D = torch.empty((M, P), dtype=torch.float32, device=A.device)
    check(ft_b2b_gemm_fwd(M, N, K, P, _dt(A), _ptr(A), _ptr(B), _ptr(C), _ptr(D), _stream_ptr(stream)))
    return D
