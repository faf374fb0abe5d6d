"""Per-step timeline of the DSMEM cluster kernel (development aid; needs build/trace/libft_trace.so).

    python tools/cluster_events.py [CTA]   (C2; CTA 0 = layer 0 slab 0)
"""
import ctypes, os, sys
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
ft.LIB_PATH = os.path.abspath("build/trace/libft_trace.so")
L = ft.lib()
L.ft_debug_cluster_events.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int]
cta = int(sys.argv[1]) if len(sys.argv) > 1 else 0
c = ftgen.CONFIGS["C2"]
p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
T = c["seq"]
buf = (ctypes.c_ulonglong * (T * 8))()
L.ft_debug_cluster_events(buf, T, cta)  # select the CTA
for _ in range(3):
    ft.stacked_lstm(*a)
torch.cuda.synchronize()
L.ft_debug_cluster_events(buf, T, cta)
ev = np.array(buf[:], dtype=np.float64).reshape(T, 8)
t0 = ev[ev > 0].min()
ev = np.where(ev > 0, (ev - t0) / 1000.0, np.nan)
names = ["hfull", "commit", "tfull", "math", "sent", "xready"]
print("step " + " ".join(f"{n:>8s}" for n in names))
for t in list(range(0, 6)) + list(range(T // 2, T // 2 + 4)) + [T - 1]:
    print(f"{t:4d} " + " ".join(f"{ev[t, k]:8.2f}" for k in range(6)))
st = np.diff(ev[:, 2])
print(f"tfull-to-tfull per step: median {np.nanmedian(st):.2f} us")
for k, n in [(0, "hfull-sent(t-1)"), (1, "commit-hfull"), (2, "tfull-commit"), (3, "math-tfull"), (4, "sent-math")]:
    if k == 0:
        v = ev[1:, 0] - ev[:-1, 4]
    else:
        v = ev[:, k] - ev[:, k - 1] if k != 2 else ev[:, 2] - ev[:, 1]
    print(f"  {n:18s} median {np.nanmedian(v):6.2f} us")
print(f"  x-ready lag behind hfull: median {np.nanmedian(ev[1:, 5] - ev[1:, 0]):6.2f} us")
