"""Per-layer timeline of the DSMEM cluster kernel (development aid; needs build/trace/libft_trace.so):
when each layer's slice-0 epilogue saw the accumulator of step t, one launch, all layers.

    python tools/cluster_layers.py [C2]
"""
import ctypes, os, sys
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
ft.LIB_PATH = os.path.abspath("build/trace/libft_trace.so")
L = ft.lib()
L.ft_debug_cluster_layer_events.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int]
c = ftgen.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
D, T = c["depth"], c["seq"]
for _ in range(3):
    ft.stacked_lstm(*a)
torch.cuda.synchronize()
s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s0.record(); ft.stacked_lstm(*a); s1.record(); torch.cuda.synchronize()
print("launch", ft.ft_last_launch(), f"{s0.elapsed_time(s1) * 1000:.1f} us (event)")
buf = (ctypes.c_ulonglong * (D * T))()
L.ft_debug_cluster_layer_events(buf, D, T)
ev = np.array(buf[:], dtype=np.float64).reshape(D, T)
t0 = ev.min()
ev = (ev - t0) / 1000.0
print("layer  t=0     t=1     t=T-1   step(median)  lag behind layer below at t=0 / median over t")
for d in range(D):
    st = np.median(np.diff(ev[d]))
    lag = ev[d] - ev[d - 1] if d else np.zeros(T)
    print(f"{d:5d} {ev[d,0]:7.2f} {ev[d,1]:7.2f} {ev[d,-1]:7.2f} {st:8.2f}      {lag[0]:6.2f} / {np.median(lag):6.2f}")
print(f"first accumulator -> last: {ev[-1,-1] - ev[0,0]:.1f} us")
