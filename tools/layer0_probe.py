"""Layer-0 chain probe (development aid): a dilated nest whose only real recurrence is layer 0
(dilations [1, T, T, ...]), C4's shape otherwise; prints ms per forward (pipelined) and the launch.
    python tools/layer0_probe.py [D]"""
import os, sys
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
D = int(sys.argv[1]) if len(sys.argv) > 1 else 2
B, T, H = 256, 100, 512
p = ftgen.stacked_inputs(B, T, H, D, 1, "bf16")
a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
dil = [1] + [T] * (D - 1)
ws = ft.Workspace()
fn = lambda: ft.stacked_lstm(*a, dilations=dil, workspace=ws)
for _ in range(5): fn()
torch.cuda.synchronize()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
reps = 30
s.record()
for _ in range(reps): fn()
e.record(); torch.cuda.synchronize()
ms = s.elapsed_time(e) / reps
print(f"D={D} dil={dil[:3]}.. {ms:.4f} ms/forward = {ms * 1000 / T:.2f} us per layer-0 step | {ft.ft_last_launch()}")
