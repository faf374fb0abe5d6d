"""C4 critical-chain analysis from the per-tile event trace (gpurun_out/events_c4.npy, written by
tools/event_run.py C4 32): per layer-0 step t, R(t) = last release of cell (0, t)'s tiles,
M(t) = last MMA-done; the step splits into R(t-1) -> M(t) (flag + loads + MMA) and M(t) -> R(t)."""
import sys
import numpy as np
sys.path.insert(0, ".")
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
ev = np.load("gpurun_out/events_c4.npy")
D, T, NT = 6, 100, 16
cells = ft.ft_wavefront_cells(0, D, T)
t0 = ev[ev > 0].min()
ev = (ev - t0) / 1000.0
R, M, S = {}, {}, {}
for g in range(len(cells) * NT):
    k, d, t, _ = cells[g // NT]
    R[(d, t)] = max(R.get((d, t), 0), ev[g, 4])
    M[(d, t)] = max(M.get((d, t), 0), ev[g, 3])
    S[(d, t)] = min(S.get((d, t), 1e18), ev[g, 0])
a = np.array([M[(0, t)] - R[(0, t - 1)] for t in range(1, T)])
b = np.array([R[(0, t)] - M[(0, t)] for t in range(1, T)])
st = np.array([R[(0, t)] - R[(0, t - 1)] for t in range(1, T)])
print(f"total {max(R.values()):.1f} us; layer-0 chain end {R[(0, T-1)]:.1f} us; top layer end {R[(D-1, T-1)]:.1f}")
print(f"layer-0 step {np.median(st):.2f} us (median) = release(t-1)->mma done(t) {np.median(a):.2f} + mma done->release {np.median(b):.2f}")
late = np.array([S[(0, t)] - R[(0, t - 1)] for t in range(1, T)])
print(f"tile of (0,t) started (producer) relative to R(t-1): median {np.median(late):.2f} us (negative = early)")
for d in range(D):
    print(f"layer {d}: last release {R[(d, T-1)]:.1f} us")
E2 = {}
for g in range(len(cells) * NT):
    k, d, t, _ = cells[g // NT]
    if d == 0:
        E2[t] = max(E2.get(t, 0), ev[g, 2])
c = np.array([E2[t] - R[(0, t - 1)] for t in range(1, T)])
e = np.array([M[(0, t)] - E2[t] for t in range(1, T)])
print(f"layer 0: release(t-1) -> last h-load issued(t) {np.median(c):.2f} us; -> mma done {np.median(e):.2f} us")
E5, E6, E7 = {}, {}, {}
for g in range(len(cells) * NT):
    k, d, t, _ = cells[g // NT]
    if d == 0:
        E5[t] = max(E5.get(t, 0), ev[g, 5]); E6[t] = max(E6.get(t, 0), ev[g, 6]); E7[t] = max(E7.get(t, 0), ev[g, 7])
f = lambda X: np.median(np.array([X[t] - R[(0, t - 1)] for t in range(1, T)]))
Mt = {t: M[(0, t)] for t in range(T)}
print(f"layer 0, relative to release(t-1): flag acquired {f(E5):.2f}, accumulator free {f(E6):.2f}, h loads issued {f(E2):.2f}, last MMA issued {f(E7):.2f}, MMA done {f(Mt):.2f} us")
rows = []
for g in range(len(cells) * NT):
    k, d, t, _ = cells[g // NT]
    if d == 0 and t >= 1:
        rows.append(ev[g] - R[(0, t - 1)])
rows = np.array(rows)
names = ["0 tile start", "1 first seg", "2 loads issued", "3 epi saw tfull", "4 released", "5 flag acq", "6 acc free", "7 last mma"]
print("per layer-0 tile, median rel. to release(t-1):", ", ".join(f"{n} {np.median(rows[:, i]):.2f}" for i, n in enumerate(names)))
print("p10:", ", ".join(f"{np.percentile(rows[:, i], 10):.2f}" for i in range(8)))
print("p90:", ", ".join(f"{np.percentile(rows[:, i], 90):.2f}" for i in range(8)))
