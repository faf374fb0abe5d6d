"""Per-tile event timeline of one stacked forward under a (band, skew) order (development aid).

usage: python tools/band_events.py CONFIG UNITS [ENV=VAL ...]   (needs build/trace/libft_trace.so)
Prints, per band, the mean per-diagonal anatomy of the critical chain:
  dep   = last producer release -> this tile's acquire returned (event 5)
  load  = acquire -> last MMA issued (event 7)
  mma   = last MMA issued -> accumulator ready (event 3)
  epi   = accumulator ready -> counter released (event 4)
and the time per band-diagonal (release of the diagonal's last cell, successive differences).
"""
import ctypes, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)) + "/..")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft

name, units = sys.argv[1], int(sys.argv[2])
band = skew = None
for kv in sys.argv[3:]:
    k, v = kv.split("=")
    os.environ[k] = v
band = int(os.environ.get("FT_BAND", "0"))
skew = int(os.environ.get("FT_SKEW", "1"))
ft.LIB_PATH = os.path.abspath("build/trace/libft_trace.so")
L = ft.lib()
c = ftgen.CONFIGS[name]
B, T, H, D = c["batch"], c["seq"], c["hidden"], c["depth"]
p = ftgen.stacked_inputs(B, T, H, D, 1, "bf16")
a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
ws = ft.Workspace()
for _ in range(4):
    ft.stacked_lstm(*a, workspace=ws)
torch.cuda.synchronize()
NT = H // units
cells = ft.ft_wavefront_cells_banded(0, D, T, 1, band, skew)
ntiles = len(cells) * NT
owner = os.environ.get("FT_OWNER", "1") != "0" and band > 0
if owner:  # owner-computes walk: events are indexed by cell_lin * NT + n (d-major, then t)
    cells = [((d // band) * (T + skew * band) + t + skew * (d % band), d, t, 0) for d in range(D) for t in range(T)]
EV_K = 8
buf = (ctypes.c_ulonglong * (ntiles * EV_K))()
L.ft_debug_events.argtypes = [ctypes.c_void_p, ctypes.c_int]
L.ft_debug_events(buf, ntiles)
ev = np.array(buf[:], dtype=np.float64).reshape(ntiles, EV_K)
t0 = ev[ev > 0].min()
ev = (ev - t0) / 1000.0
rel, cell_of = {}, []
for g in range(ntiles):
    k, d, t, _ = cells[g // NT]
    cell_of.append((k, d, t))
    rel[(d, t)] = max(rel.get((d, t), 0.0), ev[g, 4])
print(f"{name} units={units} band={band} skew={skew} owner={owner}: span {ev[:, 4].max():.1f} us, {ntiles} tiles")
bw = band if 0 < band < D else D
stats = {}
for g in range(ntiles):
    k, d, t = cell_of[g]
    deps = ([rel[(d - 1, t)]] if d > 0 else []) + ([rel[(d, t - 1)]] if t > 0 else [])
    ready = max(deps) if deps else 0.0
    s = stats.setdefault(d // bw, [])
    s.append((ev[g, 5] - ready if deps else np.nan, ev[g, 7] - max(ev[g, 5], ready), ev[g, 3] - ev[g, 7],
              ev[g, 4] - ev[g, 3], ev[g, 3] - ev[g, 6]))
for b_, s in sorted(stats.items()):
    s = np.array(s)
    print(f" band {b_}: dep {np.nanmean(s[:, 0]):.2f}  load {np.mean(s[:, 1]):.2f}  mma {np.mean(s[:, 2]):.2f}"
          f"  epi {np.mean(s[:, 3]):.2f}  (acc->ready {np.mean(s[:, 4]):.2f}) us")
# per band-diagonal completion times
diag_end = {}
for (k, d, t) in set(cell_of):
    diag_end[k] = max(diag_end.get(k, 0.0), rel[(d, t)])
ks = sorted(diag_end)
steps = np.diff([diag_end[k] for k in ks])
print(f" per-diagonal: median {np.median(steps):.2f} us, mean {np.mean(steps):.2f} us over {len(ks)} diagonals")
np.save(f"gpurun_out/bandev_{name}_{band}_{skew}_{units}.npy", ev)
