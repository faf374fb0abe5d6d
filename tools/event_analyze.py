"""Analyse the per-tile event timeline of C3 (gpurun_out/events_c3.npy)."""
import sys
import numpy as np
sys.path.insert(0, ".")
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
ev = np.load(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/events_c3.npy")
D, T, NT = (int(v) for v in (sys.argv[2:5] if len(sys.argv) > 4 else (16, 100, 16)))
dil = [int(v) for v in sys.argv[5].split(",")] if len(sys.argv) > 5 else [1] * D
npairs = 74
cells = ft.ft_wavefront_cells(0, D, T)  # order
t0 = ev[ev > 0].min()
ev = (ev - t0) / 1000.0  # us
ntiles = len(cells) * NT
tile_cell = [cells[g // NT] for g in range(ntiles)]
rel = {}
mma = {}
for g in range(ntiles):
    k, d, t, _ = tile_cell[g]
    rel[(d, t)] = max(rel.get((d, t), 0), ev[g, 4])
    mma[(d, t)] = max(mma.get((d, t), 0), ev[g, 3])
print(f"total span {ev[:, 4].max():.1f} us")
# per tile: dependency ready time vs wait start
waits, lates = [], []
bydiag = {}
for g in range(ntiles):
    k, d, t, _ = tile_cell[g]
    deps = []
    if d > 0: deps.append(rel[(d - 1, t)])
    if t >= dil[d]: deps.append(rel[(d, t - dil[d])])
    ready = max(deps) if deps else 0
    w = ev[g, 1] - ev[g, 0]
    waits.append(w)
    bydiag.setdefault(k, []).append((ev[g, 0], ev[g, 1], ev[g, 3], ev[g, 4]))
waits = np.array(waits)
print(f"dep wait per tile: mean {waits.mean():.2f} us, median {np.median(waits):.2f}, p90 {np.percentile(waits, 90):.2f}, total/pairs {waits.sum()/npairs:.0f} us")
# epilogue latency: release - mma done
epi = ev[:, 4] - ev[:, 3]
print(f"epilogue (mma done -> release) per tile: mean {epi.mean():.2f} us, p90 {np.percentile(epi, 90):.2f}")
# load+mma latency: mma done - deps ready
lm = ev[:, 3] - ev[:, 1]
print(f"deps ready -> mma done per tile: mean {lm.mean():.2f} us, p10 {np.percentile(lm,10):.2f} p90 {np.percentile(lm, 90):.2f}")
# per diagonal completion times
print("diag: first-start  last-release  (span)")
prev = 0
for k in sorted(bydiag):
    arr = np.array(bydiag[k])
    if k < 8 or k > (T + D - 8) or k % 10 == 0:
        print(f"  {k:3d}: start {arr[:,0].min():8.1f}  ready {arr[:,1].min():8.1f}..{arr[:,1].max():8.1f}  release {arr[:,3].max():8.1f}")
# where does each pair wait? fraction of dep-wait in ramp (k<16 or k>=T-1) vs steady
ks = np.array([tile_cell[g][0] for g in range(ntiles)])
ramp = (ks < D) | (ks >= T - 1)
print(f"dep wait share: ramp {waits[ramp].sum()/waits.sum()*100:.0f}%  steady {waits[~ramp].sum()/waits.sum()*100:.0f}%")
