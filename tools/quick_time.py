"""Quick device timing of the forward (development aid; bench.py is the contract)."""
import sys, time, json, os
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft

def timeit(fn, reps=10, warm=3):
    """Per call with the GPU idle before each call (includes the call's host-side latency: ctypes,
    validation, counter reset, launch), and pipelined: `reps` calls back to back between two events
    (the device time per forward of a serving loop whose host enqueues ahead of the GPU)."""
    for _ in range(warm): fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(reps):
        s.record(); fn(); e.record(); torch.cuda.synchronize(); ts.append(s.elapsed_time(e))
    s.record()
    for _ in range(reps): fn()
    e.record(); torch.cuda.synchronize()
    return float(np.median(ts)), float(np.min(ts)), s.elapsed_time(e) / reps

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)) + "/..")
import bench
res = {}
for name in sys.argv[1:] or ["C2", "C3", "C4", "C5"]:
    if ":" in name:  # custom stacked spec  name:B,T,H,D
        B_, T_, H_, D_ = (int(v) for v in name.split(":")[1].split(","))
        c = dict(kind="stacked", batch=B_, seq=T_, hidden=H_, depth=D_)
    else:
        c = ftgen.CONFIGS[name]
    ws = ft.Workspace()
    if c["kind"] == "grid":
        g = ftgen.grid_inputs(c["batch"], c["len_x"], c["len_y"], c["hidden"], c["depth"], 1, "bf16")
        a = [torch.from_numpy(g[k]).cuda().to(torch.bfloat16) for k in ("x","ys","W","U")] + [torch.from_numpy(g["b"]).cuda()]
        fn = lambda: ft.grid_rnn(*a, workspace=ws)
        flops = 48 * c["hidden"]**2 * c["len_x"] * c["len_y"] * c["depth"] * c["batch"]
    else:
        p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
        a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x","W","U")] + [torch.from_numpy(p["b"]).cuda()]
        dil = list(c.get("dilations", [])) or None
        fn = lambda: ft.stacked_lstm(*a, dilations=dil, workspace=ws)
        H, T, D, B = c["hidden"], c["seq"], c["depth"], c["batch"]
        if dil:
            flops = sum(2*B*4*H*(H*T + H*max(0, T-s)) for s in dil)
        else:
            flops = 16 * H * H * T * D * B
    if os.environ.get("QT_GRAPH") == "1":  # the forward captured once into a CUDA graph, replayed
        fn()
        torch.cuda.synchronize()
        gr = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gr):
            fn()
        fn = gr.replay
    cs = bench.ClockSampler(0)
    cs.start()
    med, mn, pipe = timeit(fn, reps=int(os.environ.get("QT_REPS", "10")), warm=int(os.environ.get("QT_WARM", "3")))
    clk = cs.stop()
    res[name] = dict(ms_median=med, ms_min=mn, ms_pipelined=pipe, tflops=flops / med / 1e9, seq_per_s=c["batch"] / med * 1e3,
                     sm_mhz=(clk or {}).get("sm_mhz"), power_w=(clk or {}).get("power_w_median"))
    print(name, json.dumps(res[name]), flush=True)
