"""C4 under the layer-0 owner walk (trace build): does the rest of the nest keep pace with layer 0?
Per layer d and step t, R(d, t) = last counter release of the cell's tiles; prints each layer's
median lag behind layer 0 (R(d, t) − R(0, t)), its growth over the run, and the layer-0 step.

    python tools/c4_layers.py      (needs build/trace/libft_trace.so, tools/trace_build.sh)
"""
import ctypes, os, sys
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
ft.LIB_PATH = os.path.abspath("build/trace/libft_trace.so")
L = ft.lib()
c = ftgen.CONFIGS["C4"]
p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
dil = list(c["dilations"])
ws = ft.Workspace()
for _ in range(4):
    ft.stacked_lstm(*a, workspace=ws, dilations=dil)
torch.cuda.synchronize()
print(ft.ft_last_launch())
D, T, H = c["depth"], c["seq"], c["hidden"]
NT = H // 64
last = ft.ft_last_launch()
mode3 = "owner=3" in last
nt0 = int(last.split("nt0=")[1].split()[0]) if "nt0=" in last else NT
EVK = 16
R = np.full((D, T), np.nan)
S = np.full((D, T), np.nan)   # first "wait start" of the cell's tiles
if mode3:  # every tile traced at cell_lin(d, t) * max(NT, nt0) + n
    Wd = max(NT, nt0)
    n = D * T * Wd
    buf = (ctypes.c_ulonglong * (n * EVK))()
    L.ft_debug_events.argtypes = [ctypes.c_void_p, ctypes.c_int]
    L.ft_debug_events(buf, n)
    ev = np.array(buf[:], dtype=np.float64).reshape(D, T, Wd, EVK)
    ev = np.where(ev > 0, (ev - ev[ev > 0].min()) / 1000.0, np.nan)
    for d in range(D):
        k = nt0 if d == 0 else NT
        R[d] = np.nanmax(ev[d, :, :k, 4], axis=1)
        S[d] = np.nanmin(ev[d, :, :k, 0], axis=1)
    # layer-0 step anatomy (events relative to R(0, t-1)): 5 flag seen, 2 loads issued, 3 MMA done
    t = np.arange(1, T)
    for kk, name in ((5, "recurrent flag seen"), (2, "A loads issued"), (3, "MMA done (epilogue saw tfull)"), (4, "released")):
        v = np.nanmax(ev[0, 1:, :nt0, kk], axis=1) - R[0, :-1]
        print(f"  layer-0 step: {name:32s} +{np.nanmedian(v):5.2f} us after R(0, t-1)")
else:
    cells = ft.ft_wavefront_cells(0, D, T)
    ncells = len(cells)
    n = ncells * NT + T * NT
    buf = (ctypes.c_ulonglong * (n * EVK))()
    L.ft_debug_events.argtypes = [ctypes.c_void_p, ctypes.c_int]
    L.ft_debug_events(buf, n)
    ev = np.array(buf[:], dtype=np.float64).reshape(n, EVK)
    ev = np.where(ev > 0, (ev - ev[ev > 0].min()) / 1000.0, np.nan)
    for g in range(ncells * NT):
        _, d, t, _ = cells[g // NT]
        if d == 0:
            continue
        R[d, t] = np.nanmax([R[d, t], ev[g, 4]])
        S[d, t] = np.nanmin([S[d, t], ev[g, 0]])
    for t in range(T):
        blk = ev[ncells * NT + t * NT: ncells * NT + (t + 1) * NT]
        R[0, t] = np.nanmax(blk[:, 4])
        S[0, t] = np.nanmin(blk[:, 0])
print(f"layer-0 step (median) {np.nanmedian(np.diff(R[0])):.2f} us; layer 0 ends {R[0, -1]:.1f} us; nest ends {np.nanmax(R):.1f} us")
for d in range(1, D):
    lag = R[d] - R[0]
    q = T // 4
    print(f"layer {d} (dil {dil[d]:2d}): lag behind layer 0 median {np.nanmedian(lag):6.2f} us, first quarter "
          f"{np.nanmedian(lag[:q]):6.2f}, last quarter {np.nanmedian(lag[-q:]):6.2f}; ends {R[d, -1]:.1f} us; "
          f"tile start -> release median {np.nanmedian(R[d] - S[d]):.2f} us")
