"""Tile-to-worker assignment of the persistent streaming kernel, simulated on the host.

The kernel enumerates tiles in the wavefront order of the product scheduler (ft_wavefront_cells,
the same __host__ __device__ code), `tiles_per_cell` consecutive tiles per cell, and worker w (a
CTA or CTA pair) processes tiles w, w + nw, w + 2nw, ... in order.  A simulation of in-order
workers that may start a tile only when its producer cells (Table 4 dependence vectors; the
dilation stride, L331) are complete must finish — the deadlock-freedom argument of DESIGN.md §6 —
and, in an event model with a dependency latency, must keep the critical path.  No GPU needed.
"""
import pytest

from paper_conf_sosp_liuqc0hs0y24_b200 import build, ft


@pytest.fixture(scope="module", autouse=True)
def _built():
    build.build()


def _producers(kind, cell, dil):
    _, d, i, j = cell
    if kind == 0:
        out = [(d - 1, i, 0)] if d > 0 else []
        if i >= dil[d]:
            out.append((d, i - dil[d], 0))
        return out
    out = [(d - 1, i, j)] if d > 0 else []
    if i > 0:
        out.append((d, i - 1, j))
    if j > 0:
        out.append((d, i, j - 1))
    return out


def _owner(ntiles, nw):
    """The kernel's static assignment: tile g of the wavefront sequence -> worker g mod nw."""
    return [g % nw for g in range(ntiles)]


def _simulate(kind, D, La, Lb, dil, tpc, nw):
    """Unit-time rounds: each worker completes its next tile when the tile's producer cells are
    complete.  Returns the number of rounds (raises on deadlock)."""
    cells = ft.ft_wavefront_cells(kind, D, La, Lb)
    ordinal = {(c[1], c[2], c[3]): o for o, c in enumerate(cells)}
    owner = _owner(len(cells) * tpc, nw)
    queues = [[] for _ in range(nw)]
    for g, w in enumerate(owner):
        assert 0 <= w < nw
        queues[w].append(g)                      # appended in g order = the worker's order
    left = [tpc] * len(cells)
    heads = [0] * nw
    rounds = 0
    remaining = len(owner)
    while remaining:
        done_now = []
        for w in range(nw):
            if heads[w] < len(queues[w]):
                g = queues[w][heads[w]]
                cell = cells[g // tpc]
                if all(left[ordinal[p]] == 0 for p in _producers(kind, cell, dil or [1] * D)):
                    done_now.append((w, g))
        assert done_now, "deadlock: no worker can make progress"
        for w, g in done_now:
            heads[w] += 1
            left[g // tpc] -= 1
        remaining -= len(done_now)
        rounds += 1
    return rounds


@pytest.mark.parametrize("kind,D,La,Lb,dil,tpc,nw", [
    (0, 6, 30, 1, [1, 2, 4, 8, 16, 32], 16, 74),   # C4-like, 32-unit tiles, 74 CTA pairs
    (0, 16, 12, 1, None, 16, 74),                   # C3-like depth, short sequence
    (0, 4, 12, 1, [1, 1, 3, 2], 8, 10),
    (0, 5, 7, 1, None, 4, 3),                       # fewer workers than tiles per cell
    (1, 3, 4, 5, None, 16, 148),                    # grid, 1-CTA workers
    (1, 4, 6, 3, None, 2, 5),
])
def test_assignment_is_deadlock_free(kind, D, La, Lb, dil, tpc, nw):
    _simulate(kind, D, La, Lb, dil, tpc, nw)


def _event_makespan(kind, D, La, Lb, dil, tpc, nw, tau=1.0, lat=2.0):
    """Event model of the persistent kernel: a worker runs its tiles in order, each takes `tau`
    (the MMA), and may start only `lat` (counter propagation + operand loads) after its producer
    cells completed.  Returns the makespan."""
    cells = ft.ft_wavefront_cells(kind, D, La, Lb)
    ordinal = {(c[1], c[2], c[3]): o for o, c in enumerate(cells)}
    owner = _owner(len(cells) * tpc, nw)
    queues = [[] for _ in range(nw)]
    for g, w in enumerate(owner):
        queues[w].append(g)
    left, end, free, heads = [tpc] * len(cells), [0.0] * len(cells), [0.0] * nw, [0] * nw
    for _ in range(len(owner)):
        best = None
        for w in range(nw):
            if heads[w] < len(queues[w]):
                g = queues[w][heads[w]]
                ps = [ordinal[p] for p in _producers(kind, cells[g // tpc], dil or [1] * D)]
                if all(left[p] == 0 for p in ps):
                    st = max([free[w]] + [end[p] + lat for p in ps])
                    if best is None or st < best[0]:
                        best = (st, w, g)
        assert best is not None, "deadlock"
        st, w, g = best
        free[w] = st + tau
        heads[w] += 1
        left[g // tpc] -= 1
        end[g // tpc] = max(end[g // tpc], st + tau)
    return max(free)


def test_assignment_keeps_the_critical_path():
    """C4's shape (6 layers, dilations 1..32, 16 tiles per cell, 74 CTA pairs) at T = 30: with
    per-tile time tau and dependency latency lat, round-robin finishes in the critical path
    (T + D - 1 steps of tau + lat) — no critical tile waits behind work that has slack.  (A
    variant reserving workers for the dilation-1 layer measured slower on the GPU: DESIGN §6.)"""
    dil = [1, 2, 4, 8, 16, 32]
    T, D, tau, lat = 30, 6, 1.0, 2.0
    span = _event_makespan(0, D, T, 1, dil, 16, 74, tau, lat)
    assert span <= (T + D - 1) * (tau + lat), span


# ------------------------------------------------------------------ layer-banded orders (kind 0)
def _banded_cells(D, T, band, skew):
    return ft.ft_wavefront_cells_banded(0, D, T, 1, band, skew)


@pytest.mark.parametrize("D,T,band,skew,dil", [
    (16, 12, 5, 2, None), (16, 12, 6, 1, None), (7, 3, 3, 2, None), (5, 1, 2, 3, None),
    (4, 9, 4, 2, None), (6, 10, 4, 2, [1, 2, 4, 8, 16, 32]), (3, 2, 1, 5, None),
])
def test_banded_order_is_a_legal_schedule(D, T, band, skew, dil):
    """Every cell exactly once; every producer (Table 4: (d-1, t) and (d, t - s_d)) strictly
    before its consumer; diagonal numbers non-decreasing; each band's cells contiguous."""
    cells = _banded_cells(D, T, band, skew)
    assert sorted((d, i) for _, d, i, _ in cells) == [(d, t) for d in range(D) for t in range(T)]
    pos = {(d, i): o for o, (_, d, i, _) in enumerate(cells)}
    dil = dil or [1] * D
    for (d, t), o in pos.items():
        if d > 0:
            assert pos[(d - 1, t)] < o
        if t >= dil[d]:
            assert pos[(d, t - dil[d])] < o
    ks = [k for k, _, _, _ in cells]
    assert ks == sorted(ks)
    bw = band if 0 < band < D else D
    bands = [d // bw for _, d, _, _ in cells]
    assert bands == sorted(bands)
    # inside a band, the diagonal of (d, t) is t + skew·(d - d0) (+ the band's offset)
    for k, d, t, _ in cells:
        d0 = (d // bw) * bw
        first_k = min(kk for kk, dd, _, _ in cells if dd // bw == d // bw)
        assert k - first_k == t + max(skew, 1) * (d - d0)


def test_banded_defaults_equal_the_paper_order():
    for D, T in [(16, 12), (3, 7), (5, 1), (1, 4)]:
        ref = ft.ft_wavefront_cells(0, D, T)
        assert _banded_cells(D, T, 0, 1) == ref
        assert _banded_cells(D, T, D, 1) == ref
        assert _banded_cells(D, T, D + 3, 0) == ref


def _simulate_cells(cells, dil, tpc, nw):
    ordinal = {(c[1], c[2]): o for o, c in enumerate(cells)}
    queues = [[] for _ in range(nw)]
    for g in range(len(cells) * tpc):
        queues[g % nw].append(g)
    left, heads, remaining = [tpc] * len(cells), [0] * nw, len(cells) * tpc
    while remaining:
        done = []
        for w in range(nw):
            if heads[w] < len(queues[w]):
                g = queues[w][heads[w]]
                _, d, t, _ = cells[g // tpc]
                ps = ([(d - 1, t)] if d > 0 else []) + ([(d, t - dil[d])] if t >= dil[d] else [])
                if all(left[ordinal[p]] == 0 for p in ps):
                    done.append((w, g))
        assert done, "deadlock"
        for w, g in done:
            heads[w] += 1
            left[g // tpc] -= 1
        remaining -= len(done)


@pytest.mark.parametrize("D,T,band,skew,tpc,nw", [
    (16, 10, 5, 2, 16, 74), (16, 10, 6, 1, 32, 74), (8, 6, 3, 2, 4, 5), (6, 9, 4, 3, 8, 148),
])
def test_banded_assignment_is_deadlock_free(D, T, band, skew, tpc, nw):
    _simulate_cells(_banded_cells(D, T, band, skew), [1] * D, tpc, nw)


# ------------------------------------------------------------ the bf16 kernel's per-worker walks
def _walks(D, T, band, skew, owner, nt, nw):
    return [ft.ft_tile_walk(D, T, band, skew, owner, nt, w, nw) for w in range(nw)]


@pytest.mark.parametrize("D,T,band,skew,nt,nw", [
    (16, 9, 4, 1, 16, 74), (7, 5, 3, 1, 4, 13), (6, 4, 4, 2, 2, 9), (5, 6, 2, 1, 3, 6),
])
def test_owner_walk_covers_every_tile_once_in_dependence_order(D, T, band, skew, nt, nw):
    """Owner-computes: every (d, t, n) exactly once; a worker keeps one slab (n, layer within
    the band) and runs t ascending inside a band, bands ascending."""
    walks = _walks(D, T, band, skew, 1, nt, nw)
    allt = sorted(x for w in walks for x in w)
    assert allt == [(d, t, n) for d in range(D) for t in range(T) for n in range(nt)]
    for w, seq in enumerate(walks):
        if w >= band * nt:
            assert seq == []
            continue
        assert len({n for _, _, n in seq}) <= 1 and len({d % band for d, _, _ in seq}) <= 1
        assert seq == sorted(seq, key=lambda x: (x[0] // band, x[1]))


@pytest.mark.parametrize("owner", [0, 1])
def test_walks_are_deadlock_free(owner):
    """Workers run their walks in order; a tile may complete when its producer cells (d-1, t)
    and (d, t-1) are complete (all N-tiles).  Must terminate for both assignments."""
    D, T, band, nt, nw = 12, 7, 4, 8, 37
    walks = _walks(D, T, band, 1, owner, nt, nw)
    left = {(d, t): nt for d in range(D) for t in range(T)}
    heads = [0] * nw
    while any(heads[w] < len(walks[w]) for w in range(nw)):
        done = []
        for w in range(nw):
            if heads[w] < len(walks[w]):
                d, t, n = walks[w][heads[w]]
                if (d == 0 or left[(d - 1, t)] == 0) and (t == 0 or left[(d, t - 1)] == 0):
                    done.append(w)
        assert done, "deadlock"
        for w in done:
            d, t, n = walks[w][heads[w]]
            heads[w] += 1
            left[(d, t)] -= 1


def test_round_robin_walk_matches_the_cell_order():
    D, T, band, nt, nw = 8, 5, 3, 4, 7
    cells = ft.ft_wavefront_cells_banded(0, D, T, 1, band, 1)
    seq = [(c[1], c[2], n) for c in cells for n in range(nt)]
    for w in range(nw):
        assert ft.ft_tile_walk(D, T, band, 1, 0, nt, w, nw) == seq[w::nw]


@pytest.mark.parametrize("D,T,nt,nw,dil", [
    (6, 12, 16, 74, [1, 2, 4, 8, 16, 32]), (3, 7, 4, 11, [1, 3, 2]), (4, 5, 2, 5, [1, 1, 2, 1]),
])
def test_layer0_owner_walk(D, T, nt, nw, dil):
    """Owner mode 2 (dilated nests): workers < nt own layer 0's N-tiles for every t; the rest
    take the other tiles round-robin in wavefront order.  Coverage, order, deadlock freedom
    with the dilated dependences (d-1, t) and (d, t - s_d)."""
    walks = [ft.ft_tile_walk(D, T, 0, 1, 2, nt, w, nw) for w in range(nw)]
    allt = sorted(x for w in walks for x in w)
    assert allt == [(d, t, n) for d in range(D) for t in range(T) for n in range(nt)]
    for w in range(nt):
        assert walks[w] == [(0, t, w) for t in range(T)]
    cells = ft.ft_wavefront_cells(0, D, T)
    order = {(c[1], c[2], n): i for i, c in enumerate(cells) for n in range(nt)}
    rest = sorted((x for w in walks[nt:] for x in w), key=lambda x: (order[x], x[2]))
    assert rest == [x for x in sorted(order, key=lambda x: (order[x], x[2])) if x[0] > 0]
    for w in range(nt, nw):
        assert walks[w] == rest[w - nt::nw - nt]
    left = {(d, t): nt for d in range(D) for t in range(T)}
    heads = [0] * nw
    while any(heads[w] < len(walks[w]) for w in range(nw)):
        done = []
        for w in range(nw):
            if heads[w] < len(walks[w]):
                d, t, n = walks[w][heads[w]]
                if (d == 0 or left[(d - 1, t)] == 0) and (t < dil[d] or left[(d, t - dil[d])] == 0):
                    done.append(w)
        assert done, "deadlock"
        for w in done:
            d, t, n = walks[w][heads[w]]
            heads[w] += 1
            left[(d, t)] -= 1


@pytest.mark.parametrize("D,T,nt,nw,dil", [
    (6, 12, 8, 74, [1, 2, 4, 8, 16, 32]), (3, 7, 4, 13, [1, 3, 2]), (4, 5, 2, 9, [1, 1, 2, 1]),
])
def test_all_layers_owner_walk(D, T, nt, nw, dil):
    """Owner mode 3 (dilated nests, D·nt <= workers): worker w owns (layer w // nt, N-tile
    w % nt) for t ascending; workers past D·nt are idle.  Coverage and deadlock freedom with the
    dilated dependences (d-1, t) and (d, t - s_d); too few workers fall back to the round-robin
    walk."""
    walks = [ft.ft_tile_walk(D, T, 0, 1, 3, nt, w, nw) for w in range(nw)]
    allt = sorted(x for w in walks for x in w)
    assert allt == [(d, t, n) for d in range(D) for t in range(T) for n in range(nt)]
    for w in range(nw):
        assert walks[w] == ([(w // nt, t, w % nt) for t in range(T)] if w < D * nt else [])
    left = {(d, t): nt for d in range(D) for t in range(T)}
    heads = [0] * nw
    while any(heads[w] < len(walks[w]) for w in range(nw)):
        done = []
        for w in range(nw):
            if heads[w] < len(walks[w]):
                d, t, n = walks[w][heads[w]]
                if (d == 0 or left[(d - 1, t)] == 0) and (t < dil[d] or left[(d, t - dil[d])] == 0):
                    done.append(w)
        assert done, "deadlock"
        for w in done:
            d, t, n = walks[w][heads[w]]
            heads[w] += 1
            left[(d, t)] -= 1
    assert ft.ft_tile_walk(D, T, 0, 1, 3, nt, 0, D * nt - 1) == ft.ft_tile_walk(D, T, 0, 1, 0, nt, 0, D * nt - 1)


@pytest.mark.parametrize("D,T,nt,nw,dil", [
    (6, 12, 8, 74, [1, 2, 4, 8, 16, 32]), (3, 7, 4, 17, [1, 3, 2]), (4, 5, 2, 11, [1, 1, 2, 1]),
])
def test_all_layers_owner_walk_narrow_layer0(D, T, nt, nw, dil):
    """Owner mode 3 with layer 0 in half-width slabs (owner code 4): workers < 2·nt own layer 0's
    half-width N-tiles, the next (D-1)·nt the other layers' slabs.  Every layer-0 half tile and
    every other (d, t, n) exactly once; deadlock-free when a cell completes after all of its
    tiles (2·nt on layer 0)."""
    walks = [ft.ft_tile_walk(D, T, 0, 1, 4, nt, w, nw) for w in range(nw)]
    allt = sorted(x for w in walks for x in w)
    want = sorted([(0, t, n) for t in range(T) for n in range(2 * nt)] +
                  [(d, t, n) for d in range(1, D) for t in range(T) for n in range(nt)])
    assert allt == want
    for w in range(nw):
        if w < 2 * nt:
            assert walks[w] == [(0, t, w) for t in range(T)]
        elif w < 2 * nt + (D - 1) * nt:
            e, n = 1 + (w - 2 * nt) // nt, (w - 2 * nt) % nt
            assert walks[w] == [(e, t, n) for t in range(T)]
        else:
            assert walks[w] == []
    left = {(d, t): (2 * nt if d == 0 else nt) for d in range(D) for t in range(T)}
    heads = [0] * nw
    while any(heads[w] < len(walks[w]) for w in range(nw)):
        done = []
        for w in range(nw):
            if heads[w] < len(walks[w]):
                d, t, n = walks[w][heads[w]]
                if (d == 0 or left[(d - 1, t)] == 0) and (t < dil[d] or left[(d, t - dil[d])] == 0):
                    done.append(w)
        assert done, "deadlock"
        for w in done:
            d, t, n = walks[w][heads[w]]
            heads[w] += 1
            left[(d, t)] -= 1


@pytest.mark.parametrize("D,Lx,Ly,band", [(4, 3, 4, 1), (4, 5, 2, 2), (5, 4, 4, 3), (3, 1, 6, 1), (2, 6, 1, 1)])
def test_grid_depth_bands_are_legal(D, Lx, Ly, band):
    """Grid nests in depth bands (band after band, each a wavefront over i + j + (d - d0)): every
    cell once, producers (d-1,i,j), (d,i-1,j), (d,i,j-1) strictly earlier, bands contiguous;
    band >= D is the paper order."""
    cells = ft.ft_wavefront_cells_banded(1, D, Lx, Ly, band, 1)
    assert sorted((c[1], c[2], c[3]) for c in cells) == [(d, i, j) for d in range(D) for i in range(Lx) for j in range(Ly)]
    pos = {(c[1], c[2], c[3]): o for o, c in enumerate(cells)}
    for (d, i, j), o in pos.items():
        for q in ((d - 1, i, j), (d, i - 1, j), (d, i, j - 1)):
            if min(q) >= 0:
                assert pos[q] < o
    bands = [c[1] // band for c in cells]
    assert bands == sorted(bands)
    assert ft.ft_wavefront_cells_banded(1, D, Lx, Ly, D, 1) == ft.ft_wavefront_cells(1, D, Lx, Ly)


# ------------------------------------------------------------------ SSA slot rings (a6)
def _simulate_ssa_rings(D, T, dil, band, seed):
    """Random legal executions of the nest against the kernel's hb slot layout (ft_ssa_slots).
    Events: start(d,t) reads h(d-1,t) and h(d,t-s) from their slots (needs both producers
    ended); end(d,t) writes h(d,t) into its slot, and — as run_epilogue does — waits first for
    the depth consumer (d+1, t-len) of the slot's previous step when the slot wraps.  Every read
    must find the step it expects; every event order the dependences allow is possible, so this
    covers the banded owner walk and the round-robin wavefront alike."""
    import random
    rows, off, mask = ft.ft_ssa_slots(D, T, dil, band)
    rng = random.Random(seed)
    slot = {}
    started, ended = set(), set()

    def row(d, t):
        r = off[d] + (t & mask[d])
        assert 0 <= r < rows
        return r

    def can_start(d, t):
        return ((d == 0 or (d - 1, t) in ended) and (t < dil[d] or (d, t - dil[d]) in ended))

    def can_end(d, t):
        if (d, t) not in started:
            return False
        m = mask[d]
        if m >= 0 and t > m and d + 1 < D:
            return (d + 1, t - m - 1) in ended
        return True

    cells = [(d, t) for d in range(D) for t in range(T)]
    while len(ended) < len(cells):
        enabled = [("s", c) for c in cells if c not in started and can_start(*c)]
        enabled += [("e", c) for c in cells if c in started and c not in ended and can_end(*c)]
        assert enabled, "deadlock: the back-pressure wait blocked every cell"
        kind, (d, t) = rng.choice(enabled)
        if kind == "s":
            if d > 0:
                assert slot.get(row(d - 1, t)) == (d - 1, t), ("depth read", d, t)
            if t >= dil[d]:
                assert slot.get(row(d, t - dil[d])) == (d, t - dil[d]), ("recurrent read", d, t)
            started.add((d, t))
        else:
            slot[row(d, t)] = (d, t)
            ended.add((d, t))


@pytest.mark.parametrize("D,T,dil,band", [
    (6, 17, [1] * 6, 0), (8, 13, [1] * 8, 4), (8, 13, [1] * 8, 3), (5, 21, [1] * 5, 2),
    (6, 40, [1, 2, 4, 8, 16, 32], 0), (4, 19, [3, 1, 7, 2], 0), (7, 9, [1] * 7, 2)])
def test_ssa_ring_layout_is_safe_under_every_order(D, T, dil, band):
    for seed in range(6):
        _simulate_ssa_rings(D, T, dil, band, seed)


def test_ssa_ring_layout_sizes():
    rows, off, mask = ft.ft_ssa_slots(16, 100, [1] * 16, 4)  # C3: 16·4 ring slots + 2·T
    assert rows == 16 * 4 + 200
    assert [m for m in mask].count(-1) == 3  # the boundary layers of bands 0..2
    rows, off, mask = ft.ft_ssa_slots(6, 100, [1, 2, 4, 8, 16, 32], 0)  # C4
    assert mask == [3, 3, 7, 15, 31, 63]
