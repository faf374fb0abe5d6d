"""Layer-0 step of C4 on the light trace build (-DFT_TRACE_LIGHT: events 1-5, 7, 9, 10 of the leader
CTA of each tile; no role counters): per step t, the spread of the 16 layer-0 tiles' release
times and the gap from the last release of step t to the first / last consumer seeing it.

    bash tools/ab_build.sh light -DFT_TRACE_LIGHT && FT_LIB_PATH=build/ab/libft_light.so python tools/c4_spread.py
"""
import ctypes, os, sys
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
L = ft.lib()
c = ftgen.CONFIGS["C4"]
p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
dil = list(c["dilations"])
ws = ft.Workspace()
for _ in range(4):
    ft.stacked_lstm(*a, workspace=ws, dilations=dil)
torch.cuda.synchronize()
last = ft.ft_last_launch()
print(last)
D, T, H = c["depth"], c["seq"], c["hidden"]
NT = H // 64
nt0 = int(last.split("nt0=")[1].split()[0])
Wd = max(NT, nt0)
n = D * T * Wd
EVK = 16
buf = (ctypes.c_ulonglong * (n * EVK))()
L.ft_debug_events.argtypes = [ctypes.c_void_p, ctypes.c_int]
L.ft_debug_events(buf, n)
ev = np.array(buf[:], dtype=np.float64).reshape(D, T, Wd, EVK)
ev = np.where(ev > 0, (ev - ev[ev > 0].min()) / 1000.0, np.nan)
R = ev[0, :, :nt0, 4]      # [T, nt0] release of layer-0 tile n at step t
M = ev[0, :, :nt0, 3]      # MMA done (epilogue saw tfull)
F = ev[0, :, :nt0, 5]      # flag of step t-1 seen by tile n's producer at step t
t = np.arange(1, T)
step = np.nanmax(R[1:], 1) - np.nanmax(R[:-1], 1)
spread = np.nanmax(R, 1) - np.nanmin(R, 1)
seen_first = np.nanmin(F[1:], 1) - np.nanmax(R[:-1], 1)
seen_last = np.nanmax(F[1:], 1) - np.nanmax(R[:-1], 1)
mma = np.nanmax(M[1:], 1) - np.nanmax(R[:-1], 1)
epi = np.nanmedian(R - M, 1)
print(f"layer-0 step (last release to last release): median {np.nanmedian(step):.2f} us")
print(f"release spread over the {nt0} tiles of a step: median {np.nanmedian(spread):.2f} us, p90 {np.nanpercentile(spread, 90):.2f}")
print(f"last release(t-1) -> flag seen at step t: first tile {np.nanmedian(seen_first):.2f} us, last tile {np.nanmedian(seen_last):.2f} us")
print(f"last release(t-1) -> last MMA done(t): {np.nanmedian(mma):.2f} us; MMA done -> release (per tile, median): {np.nanmedian(epi):.2f} us")
order = np.argsort(np.nanmedian(R - np.nanmin(R, 1, keepdims=True), 0))
print("tiles by median release lag:", [(int(k), round(float(np.nanmedian(R[:, k] - np.nanmin(R, 1))), 2)) for k in order])

# finer anatomy of step t (medians over t of the max over tiles), relative to the last release of t-1
names = {5: "A producer saw the flag", 8: "A producer got the slot of the first recurrent chunk",
         11: "MMA warp saw the last input-half chunk land", 9: "A producer got the slot of the last chunk", 2: "A loads issued",
         10: "MMA warp saw the first recurrent chunk land", 7: "MMA warp issued the last chunk",
         3: "epilogue saw the accumulator", 13: "epilogue: first TMEM chunk in registers",
         14: "epilogue: math and h stores issued (leader warp)", 4: "released"}
for k in (11, 5, 8, 9, 2, 10, 7, 3, 13, 14, 4):
    v = np.nanmax(ev[0, 1:, :nt0, k], 1) - np.nanmax(R[:-1], 1)
    print(f"  +{np.nanmedian(v):5.2f} us  {names[k]}")
