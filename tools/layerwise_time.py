"""NEXT-2 comparison on one B200: the one-launch wavefront (ft_stacked_lstm_fwd) vs the
layer-sequential schedule (ft_stacked_lstm_layerwise_fwd: hoisted cuBLAS input GEMM + U-resident
recurrent kernel per layer), same inputs; prints ms per forward and the normwise difference."""
import sys, json
import torch
sys.path.insert(0, ".")
import ftgen, bench
from paper_conf_sosp_liuqc0hs0y24_b200 import ft

def timeit(fn, reps):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps): fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / reps

specs = [a.split(":") for a in sys.argv[1:]] or [["C2", "64,64,256,8"], ["C3", "256,100,1024,16"],
                                                 ["C3_Bg32", "32,100,1024,16"], ["C3_Bg128", "128,100,1024,16"],
                                                 ["H256_T128_D32", "256,128,256,32"], ["H1024_T64_D8", "256,64,1024,8"]]
for name, shp in specs:
    B, T, H, D = map(int, shp.split(","))
    p = ftgen.stacked_inputs(B, T, H, D, 11, "bf16")
    x = torch.from_numpy(p["x"]).cuda().to(torch.bfloat16)
    W, U = (torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("W", "U"))
    b = torch.from_numpy(p["b"]).cuda()
    ws1, ws2 = ft.Workspace(), ft.Workspace()
    reps = 20 if B * T * H * D < 1e8 else 10
    cs = bench.ClockSampler(0); cs.start()
    wf = timeit(lambda: ft.stacked_lstm(x, W, U, b, workspace=ws1), reps)
    lw = timeit(lambda: ft.stacked_lstm_layerwise(x, W, U, b, workspace=ws2), reps)
    clk = cs.stop() or {}
    a = ft.stacked_lstm(x, W, U, b, workspace=ws1)["y"].float()
    c = ft.stacked_lstm_layerwise(x, W, U, b, workspace=ws2)["y"].float()
    diff = float((a - c).abs().max() / a.abs().max().clamp_min(1e-30))
    print(json.dumps(dict(name=name, B=B, T=T, H=H, D=D, wavefront_ms=round(wf, 4),
                          layerwise_ms=round(lw, 4), speedup=round(lw / wf, 2), y_normrel_diff=diff,
                          sm_mhz=clk.get("sm_mhz"))), flush=True)
