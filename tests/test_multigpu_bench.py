"""The N-rank bench path: `bench.py --gpus N` launches its own
N ranks, shards the batch map (weak scaling: 256 sequences per rank), runs the final output
gather inside every timed step and has rank 0 check the gathered outputs bitwise against a
recomputation of every shard (pin P12: per-row arithmetic does not depend on the shard).

gpurun gives one GPU, so the N ranks share cuda:0 (FT_BENCH_SHARED_GPU=1: gloo control plane,
fused gather over CUDA IPC inside one device).  On a node with >= N GPUs the NCCL legs run too
(one GPU per rank: torch.distributed over NCCL, the fused gather over NVLink peer memory, and
the library's ft_comm_gather_rank)."""
import json
import os
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(n, extra=(), shared=True, timeout=900):
    env = dict(os.environ)
    if shared:
        env["FT_BENCH_SHARED_GPU"] = "1"
    else:
        env.pop("FT_BENCH_SHARED_GPU", None)
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", str(n), "--steps", "2",
           "--warmup", "3", "--no-cpu-baseline", *extra]
    r = subprocess.run(cmd, env=env, cwd=ROOT, capture_output=True, text=True, timeout=timeout)
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    if r.returncode != 0:  # keep the whole log (torchrun's rank tracebacks are long)
        os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
        with open(os.path.join(ROOT, "gpurun_out", f"bench_n{n}_failed.log"), "w") as f:
            f.write(r.stdout + "\n----- stderr\n" + r.stderr)
    assert r.returncode == 0 and len(lines) == 1, (r.returncode, r.stdout[-2000:], r.stderr[-4000:])
    return json.loads(lines[0]), r


@pytest.mark.parametrize("n", [2, 4])
def test_bench_n_ranks_share_one_gpu(cuda_device, n):
    d, _ = _bench(n)
    assert d["n_gpus"] == n
    assert d["config"]["global_batch"] == 256 * n and d["config"]["per_gpu_batch"] == 256
    assert d["config"]["gather"] == "fused"
    assert d["gather_ok"] is True
    assert d["e2e"]["matches_device_path"] is True
    assert d["value"] > 0


def test_bench_refuses_more_gpus_than_visible(cuda_device):
    n = torch.cuda.device_count() + 1
    env = dict(os.environ)
    env.pop("FT_BENCH_SHARED_GPU", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", str(n), "--steps", "2",
                        "--warmup", "3"], env=env, cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 2 and not [l for l in r.stdout.splitlines() if l.startswith("{")], r.stderr[-2000:]


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs >= 2 GPUs (NCCL legs)")
@pytest.mark.parametrize("gather", ["fused", "nccl"])
def test_bench_two_gpus_nccl(cuda_device, gather):
    d, r = _bench(2, ("--gather", gather), shared=False)
    assert d["n_gpus"] == 2 and d["gather_ok"] is True and d["config"]["control_plane"] == "nccl"
    assert "nranks 2" in r.stderr.lower() or "nranks=2" in r.stderr.lower() or "nRanks 2" in r.stderr


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs >= 2 GPUs (NCCL send/recv)")
def test_comm_gather_abi_multi_device(cuda_device):
    """ft_comm_create over every visible device (one process, ncclCommInitAll) and a gather of
    each device's slice to the root — the NCCL send/recv legs of ft_comm_gather."""
    from paper_conf_sosp_liuqc0hs0y24_b200 import ft
    nd = torch.cuda.device_count()
    st, comm = ft.ft_comm_create(list(range(nd)))
    assert st == ft.FT_OK, ft.ft_last_error()
    n = 1 << 16
    srcs = [torch.full((n,), float(r + 1), device=f"cuda:{r}") + torch.arange(n, device=f"cuda:{r}")
            for r in range(nd)]
    for root in (0, nd - 1):
        dst = torch.zeros(n * nd, device=f"cuda:{root}")
        streams = [torch.cuda.current_stream(r).cuda_stream for r in range(nd)]
        st = ft.ft_comm_gather(comm, [s.data_ptr() for s in srcs], dst.data_ptr(), [n * 4] * nd, root, streams)
        assert st == ft.FT_OK, ft.ft_last_error()
        for r in range(nd):
            torch.cuda.synchronize(r)
        assert torch.equal(dst.cpu(), torch.cat([s.cpu() for s in srcs]))
    assert ft.ft_comm_destroy(comm) == ft.FT_OK
