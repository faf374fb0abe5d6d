"""C3 strong-scaling projection: the per-GPU forward time when the 256-sequence batch
is sharded over G GPUs (B_g = 256/G) — each GPU still streams the full 256 MiB weight set every
diagonal.  Device time on one GPU at each B_g (the GPUs of a batch-sharded run are independent)."""
import sys, json, os
import torch
sys.path.insert(0, ".")
import ftgen, bench
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
c = ftgen.CONFIGS["C3"]
p = ftgen.stacked_inputs(256, c["seq"], c["hidden"], c["depth"], 3, "bf16")
x = torch.from_numpy(p["x"]).cuda().to(torch.bfloat16)
W, U = (torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("W", "U"))
b = torch.from_numpy(p["b"]).cuda()
ws = ft.Workspace()
for G in (1, 2, 4, 8):
    Bg = 256 // G
    xs = x[:Bg].contiguous()
    fn = lambda: ft.stacked_lstm(xs, W, U, b, workspace=ws)
    for _ in range(5): fn()
    torch.cuda.synchronize()
    cs = bench.ClockSampler(0); cs.start()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(40): fn()
    e.record(); torch.cuda.synchronize()
    clk = cs.stop() or {}
    ms = s.elapsed_time(e) / 40
    print(json.dumps(dict(G=G, per_gpu_batch=Bg, ms=ms, strong_seq_per_s=256 / ms * 1e3,
                          weak_seq_per_s_if_256_per_gpu=None, sm_mhz=clk.get("sm_mhz"),
                          power_w=clk.get("power_w_median"))), flush=True)
