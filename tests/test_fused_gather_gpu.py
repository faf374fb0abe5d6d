"""NEXT-1: the output gather fused into the kernel (shard.PeerGather).

Two ranks (processes) share cuda:0 — gpurun gives one GPU; on an NVSwitch node the same code maps
a peer GPU's memory over NVLink.  Rank 0 allocates the full y / h_n / c_n; each rank passes its row
slice of rank 0's buffers straight to ft_stacked_lstm_fwd, so the epilogue stores land in rank 0's
memory.  The gathered result must equal a single-process run of the whole batch (rows are
independent — Table 1; both runs use the same 128-row tile shape, so bitwise)."""
import os
import socket

import pytest
import torch

pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out_path):
    import numpy as np
    import torch.distributed as dist
    import ftgen
    from paper_conf_sosp_liuqc0hs0y24_b200 import ft
    from paper_conf_sosp_liuqc0hs0y24_b200.shard import PeerGather, shard_rows
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    Bt, T, H, D = 128, 5, 128, 3
    p = ftgen.stacked_inputs(Bt, T, H, D, 4242, "bf16")
    bf = torch.bfloat16
    W, U = (torch.from_numpy(p[k]).cuda().to(bf) for k in ("W", "U"))
    b = torch.from_numpy(p["b"]).cuda()
    a, e = shard_rows(Bt, world, rank)
    x = torch.from_numpy(np.ascontiguousarray(p["x"][a:e])).cuda().to(bf)
    peer = PeerGather(Bt, T, H, D, bf, "cuda:0", dst=0)
    ft.stacked_lstm(x, W, U, b, out=peer.local())
    full = peer.done()
    if rank == 0:
        import oracle
        xf = torch.from_numpy(p["x"]).cuda().to(bf)
        ref = ft.stacked_lstm(xf, W, U, b)
        torch.cuda.synchronize()
        ok = {k: bool(torch.equal(full[k], ref[k])) for k in ("y", "h_n", "c_n")}
        # and the gathered batch against the CPU oracle (fp64) on the same seeded inputs
        ora = oracle.stacked_lstm(p["x"], p["W"], p["U"], p["b"])
        for k in ("y", "h_n", "c_n"):
            g = full[k].float().cpu().numpy().astype(np.float64)
            ok["oracle_" + k] = float(np.max(np.abs(g - ora[k])) / np.max(np.abs(ora[k])))
        with open(out_path, "w") as f:
            f.write(repr(ok))
    peer.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_fused_gather_ranks_one_gpu(world, tmp_path, cuda_device):
    """world = 3: ragged shards (43 + 43 + 42 rows) whose slices start mid-tile in rank 0's
    buffers.  Bitwise equal to the single-process run, and within the bf16 tolerance of the
    oracle."""
    import torch.multiprocessing as mp
    out = str(tmp_path / "ok.txt")
    mp.spawn(_worker, args=(world, _free_port(), out), nprocs=world, join=True)
    res = eval(open(out).read())
    assert all(res[k] is True for k in ("y", "h_n", "c_n")), res
    assert all(res["oracle_" + k] <= 2e-2 for k in ("y", "h_n", "c_n")), res


def test_comm_gather_abi_one_device(cuda_device):
    """ft_comm_create / ft_comm_gather / ft_comm_destroy on the one GPU gpurun gives: the root's
    own slice is copied into place (the NCCL send/recv leg needs >= 2 devices).  On an 8-GPU node
    the same call gathers every device's y slice to the root over NVLink."""
    from paper_conf_sosp_liuqc0hs0y24_b200 import ft
    st, comm = ft.ft_comm_create([0])
    assert st == ft.FT_OK, ft.ft_last_error()
    src = torch.arange(4096, dtype=torch.float32, device="cuda")
    dst = torch.zeros_like(src)
    s = torch.cuda.current_stream().cuda_stream
    st = ft.ft_comm_gather(comm, [src.data_ptr()], dst.data_ptr(), [src.numel() * 4], 0, [s])
    assert st == ft.FT_OK, ft.ft_last_error()
    torch.cuda.synchronize()
    assert torch.equal(src, dst)
    assert ft.ft_comm_gather(comm, [src.data_ptr()], dst.data_ptr(), [16], 1, [s]) == ft.FT_ERR_INVALID_ARGUMENT
    assert ft.ft_comm_destroy(comm) == ft.FT_OK
