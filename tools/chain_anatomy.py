"""Per-step anatomy of a single-layer chain (development aid; needs the FT_TRACE build from
tools/trace_build.sh).  For a 1-layer stacked LSTM every step t+1 waits for all N-tiles of step t,
so the step time is the critical chain.  Per step (medians over t):
  sync   R(t)   -> E5(t+1)  last producer counter observed by the consumer's activation producer
  issue  E5     -> E2       recurrent-half A loads issued
  land   E2     -> E7       loads landed + last MMA chunk issued
  tail   E7     -> E3       MMA completion seen by the epilogue
  epi    E3     -> E4       epilogue (TMEM -> math -> h stores -> release)
usage: python tools/chain_anatomy.py B T H UNITS [owner]
  owner: a 2-layer dilated nest (dilations 1, T) whose layer 0 runs on the layer-0 owners;
  the anatomy is layer 0's."""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import ftgen  # noqa: E402
from paper_conf_sosp_liuqc0hs0y24_b200 import ft  # noqa: E402

B, T, H, U = (int(v) for v in sys.argv[1:5])
OWNER = len(sys.argv) > 5 and sys.argv[5] == "owner"
os.environ["FT_TILE_UNITS"] = str(U)
os.environ["FT_RESIDENT"] = "0"
ft.LIB_PATH = os.path.abspath(os.environ.get("FT_TRACE_LIB", "build/trace/libft_trace.so"))
L = ft.lib()
p = ftgen.stacked_inputs(B, T, H, 2 if OWNER else 1, 1, "bf16")
a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
ws = ft.Workspace()
for _ in range(4):
    ft.stacked_lstm(*a, workspace=ws, dilations=[1, T] if OWNER else None)
torch.cuda.synchronize()
print(ft.ft_last_launch())
NT = H // U
EVK = 16
if OWNER:  # layer-0 owner tiles are traced at ids ncells*NT + t*NT0 + n
    NT0 = NT
    base = 2 * T * NT
    n = base + T * NT0
    buf = (ctypes.c_ulonglong * (n * EVK))()
    L.ft_debug_events.argtypes = [ctypes.c_void_p, ctypes.c_int]
    L.ft_debug_events(buf, n)
    ev = np.array(buf[:], dtype=np.float64)[base * EVK:].reshape(T, NT0, EVK)
else:
    n = T * NT
    buf = (ctypes.c_ulonglong * (n * EVK))()
    L.ft_debug_events.argtypes = [ctypes.c_void_p, ctypes.c_int]
    L.ft_debug_events(buf, n)
    ev = np.array(buf[:], dtype=np.float64).reshape(T, NT, EVK)
ev = (ev - ev[ev > 0].min()) / 1000.0
R = ev[:, :, 4].max(1)
E5, E2, E7, E3 = (ev[:, :, k].max(1) for k in (5, 2, 7, 3))
t = np.arange(1, T)
parts = {"sync": E5[t] - R[t - 1], "issue": E2[t] - E5[t], "land": E7[t] - E2[t],
         "tail": E3[t] - E7[t], "epi": R[t] - E3[t], "step": R[t] - R[t - 1]}
print(f"B={B} T={T} H={H} U={U}: " + "  ".join(f"{k} {np.median(v):.2f}" for k, v in parts.items()) + " us")
# every event of step t+1 relative to R(t) (the release that enables it)
rel = {f"E{k}": np.median(ev[t, :, k].max(1) - R[t - 1]) for k in range(16)}
rel_min = {f"E{k}": np.median(ev[t, :, k].min(1) - R[t - 1]) for k in range(16)}
print("  rel to R(t-1) max over tiles: " + " ".join(f"{k}={v:.2f}" for k, v in rel.items()))
print("  rel to R(t-1) min over tiles: " + " ".join(f"{k}={v:.2f}" for k, v in rel_min.items()))
