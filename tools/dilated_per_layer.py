"""C4 (dilated LSTM, dilations 1..32) as one wavefront launch vs layer by layer (development aid): the
layer-by-layer schedule is the same library called once per layer (a one-layer dilated nest whose
h_all feeds the next layer's x), i.e. the DAG execution of L67 that the paper's Fig. 9 compares with.
Prints ms per forward (pipelined) and the normwise difference of y."""
import sys
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft

c = ftgen.CONFIGS["C4"]
B, T, H, D = c["batch"], c["seq"], c["hidden"], c["depth"]
dil = list(c["dilations"])
p = ftgen.stacked_inputs(B, T, H, D, 1, "bf16")
x = torch.from_numpy(p["x"]).cuda().to(torch.bfloat16)
W, U = (torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("W", "U"))
b = torch.from_numpy(p["b"]).cuda()
ws = ft.Workspace()
wsl = [ft.Workspace() for _ in range(D)]


def wavefront():
    return ft.dilated_rnn(x, W, U, b, dil, workspace=ws)["y"]


def per_layer():
    a = x
    for d in range(D):
        r = ft.dilated_rnn(a, W[d:d + 1].contiguous(), U[d:d + 1].contiguous(), b[d:d + 1].contiguous(), [dil[d]],
                           workspace=wsl[d])
        a = r["y"]
    return a


def timeit(fn, reps=30):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps): fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / reps


y1, y2 = wavefront(), per_layer()
torch.cuda.synchronize()
diff = float((y1.float() - y2.float()).abs().max() / y1.float().abs().max())
tw, tl = timeit(wavefront), timeit(per_layer)
print(f"C4 wavefront {tw:.3f} ms, layer by layer ({D} launches) {tl:.3f} ms, ratio {tl / tw:.2f}x, y normwise diff {diff:.2e}")
