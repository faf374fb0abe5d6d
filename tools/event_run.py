"""Per-tile event timeline of one C3 forward (development aid): where the critical path goes."""
import ctypes, sys, os
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
ft.LIB_PATH = os.path.abspath("build/trace/libft_trace.so")
L = ft.lib()
name = sys.argv[1] if len(sys.argv) > 1 else "C3"
nt_units = int(sys.argv[2]) if len(sys.argv) > 2 else 64
c = ftgen.CONFIGS[name]
p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
ws = ft.Workspace()
dil = list(c.get("dilations", [])) or None
for _ in range(4): ft.stacked_lstm(*a, workspace=ws, dilations=dil)
torch.cuda.synchronize()
D, T, NT = c["depth"], c["seq"], c["hidden"] // nt_units
ntiles = D * T * NT
EV_K = 8
buf = (ctypes.c_ulonglong * (ntiles * EV_K))()
L.ft_debug_events.argtypes = [ctypes.c_void_p, ctypes.c_int]
L.ft_debug_events(buf, ntiles)
ev = np.array(buf[:], dtype=np.float64).reshape(ntiles, EV_K)
np.save(f"gpurun_out/events_{name.lower()}.npy", ev)
print("saved", ev.shape)
