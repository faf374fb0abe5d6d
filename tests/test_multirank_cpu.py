"""World-size-2 gloo tests of the batch-map sharding (pin P12 on the host side):
each rank runs its contiguous batch slice, the gathered outputs equal the single-process run
bitwise.  The per-rank compute here is the CPU oracle (test infrastructure) — what is under test
is the sharding / gather plumbing that bench.py uses around the GPU path."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import ftgen
import oracle
from paper_conf_sosp_liuqc0hs0y24_b200.shard import gather_rows, shard_rows


def test_shard_rows_partition():
    for total in (1, 7, 256, 257):
        for world in (1, 2, 3, 8):
            spans = [shard_rows(total, world, r) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == total
            for (a, b), (c, d) in zip(spans, spans[1:]):
                assert b == c
            sizes = [b - a for a, b in spans]
            assert max(sizes) - min(sizes) <= 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, B, out_path):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    p = ftgen.stacked_inputs(B, 5, 16, 3, 4242, "f32")
    a, b = shard_rows(B, world, rank)
    r = oracle.stacked_lstm(p["x"][a:b], p["W"], p["U"], p["b"])
    full = {k: gather_rows(torch.from_numpy(r[k]), B) for k in ("y", "h_n", "c_n")}
    if rank == 0:
        np.savez(out_path, **{k: v.numpy() for k, v in full.items()})
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("B", [6, 7])
def test_two_rank_batch_shard_gather_equals_single(tmp_path, B):
    out = str(tmp_path / "g.npz")
    mp.start_processes(_worker, args=(2, _free_port(), B, out), nprocs=2, join=True,
                       start_method="spawn")
    got = np.load(out)
    p = ftgen.stacked_inputs(B, 5, 16, 3, 4242, "f32")
    ref = oracle.stacked_lstm(p["x"], p["W"], p["U"], p["b"])
    for k in ("y", "h_n", "c_n"):
        assert np.array_equal(got[k], ref[k]), k


def test_bench_refuses_to_mislabel_gpu_count():
    """`bench.py --gpus N` never reports fewer ranks than asked: without N visible GPUs it exits 2
    before printing a JSON line; under a torchrun whose WORLD_SIZE differs it exits 2 too."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    if torch.cuda.is_available():
        pytest.skip("checks the no-device refusal")
    env = dict(os.environ)
    env.pop("FT_BENCH_SHARED_GPU", None)
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--steps", "2",
                        "--warmup", "3"], env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode == 2 and "needs 2 visible CUDA devices" in r.stderr
    assert not [l for l in r.stdout.splitlines() if l.startswith("{")]
    env.update(WORLD_SIZE="3", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--steps", "2",
                        "--warmup", "3"], env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode == 2 and "WORLD_SIZE=3 != --gpus 2" in r.stderr
