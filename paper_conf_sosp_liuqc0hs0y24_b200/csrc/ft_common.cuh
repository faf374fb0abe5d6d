// ft_common.cuh — problem description, wavefront cell order and readiness-flag protocol shared
// by every kernel of the library (host + device).  Nothing here is shared with oracle/.
//
// The schedule is the paper's reordering result (§5.2): the nest
// map(batch) ∘ scan(depth) ∘ scan(time) is fully permutable (L333–L335) with constant
// dependence distances (Table 4), so one transformed dimension — the hyperplane
// π = d + t (T's first row [0,1,1,0], L341/L349) — carries every dependence.  Cells are handed
// out diagonal by diagonal; inside a diagonal every cell is independent (Fig. 9: "cells of
// the same colour run in parallel").  The batch dimension, whose null-space carries the weight
// reuse (L345–L349), is the GEMM M dimension inside a cell.
#pragma once

#include <cstdint>

#include "../../include/ft.h"

// Result-invalidating timing experiments (FT_DEBUG bits other than the stress bit 64) exist only
// in development builds compiled with -DFT_DEV_EXPERIMENTS; in the release library the test is a
// compile-time false, so no such branch is even in the binary.
#ifdef FT_DEV_EXPERIMENTS
#define FT_DEV_BIT(dbg, bit) (((dbg) & (bit)) != 0)
#else
#define FT_DEV_BIT(dbg, bit) false
#endif

#ifdef __CUDACC__
#define FT_HD __host__ __device__ __forceinline__
#else
#define FT_HD inline
#endif

namespace ft {

enum Kind : int { KIND_SEQ = 0 /* stacked + dilated */, KIND_GRID = 1 };
// Cell function: the LSTM of Listing 2 (L607–L615) or the linear cell y = x@w + s of Listing 1
// (L165; one weight matrix, no gates, the recurrent term is an addition of the previous output).
enum CellType : int { CELL_LSTM = 0, CELL_LINEAR = 1 };

// One launch's problem.  All sizes in elements.
struct Problem {
    int kind;
    int cell;            // CellType
    int B, H, D;
    int L0, L1;          // KIND_SEQ: L0 = seq, L1 = 1.  KIND_GRID: L0 = len_x, L1 = len_y.
    int naxes;           // 1 (seq) or 2 (grid)
    int BM, BNU;         // batch rows and hidden units per tile (kernel-specific)
    int MB, NT;          // m-blocks = ceil(B/BM), n-tiles per axis = ceil(H/BNU)
    int flag_mult;       // counter increments per tile (CTAs per tile: 2 for a tcgen05 CTA pair)
    int resident_layers; // bf16: layers whose weights are kept in L2 (evict_last); others stream
    int persist_layers;  // bf16 streaming: W of the first persist_layers layers lie in a persisting
                         // L2 access-policy window (loaded with EVICT_NORMAL); host side: -1 = auto
    int debug;           // 64 = stress mode (env FT_STRESS=1): random delays before each counter
                         // release — results stay valid; tests use it to shake out ordering bugs.
                         // Development builds only (-DFT_DEV_EXPERIMENTS, env FT_DEBUG; never
                         // compiled into libft.so, results INVALID): 1 skip dependency waits,
                         // 2 skip the epilogue math/stores, 4 no MMAs, 16 no weight loads,
                         // 32 fixed load coordinates, 128 EVICT_NORMAL state
    int l2pol;           // bf16 streaming: L2 eviction-policy overrides, 2 bits each (0 default,
                         // 1 first, 2 normal, 3 last): weights | state stores << 2 | A loads << 4
    int x_direct;        // bf16 streaming: layer-0 inputs read from x [B][T][H] (host-IO overlap)
    int owner;           // KIND_SEQ tile assignment (see TileWalk): 0 round-robin, 1 owner-computes
                         // under bands, 2 layer 0 owned (dilated nests) + round-robin for the rest
    int band, skew;      // KIND_SEQ order (0 = defaults D, 1): layers are processed in bands of
                         // `band` consecutive layers, each band a wavefront π = t + skew·(d − d0)
                         // (see next_cell); bands run one after the other
    int nt0;             // owner mode 3: layer 0's N-tiles when layer 0 runs narrower slabs than
                         // the other layers (0 = NT, the same width)
    int rec_first;       // KIND_SEQ: a layer with dilation >= 2 runs its K loop recurrent half
                         // first (see segments)
    int hring;           // bf16 streaming KIND_SEQ: hb holds a ring of slots per layer instead of
                         // every (d, t) row (see hb_slot_row); 0 = one row per (d, t)
    int hb_rows;         // hring: rows of hb the workspace reserves (Σ ring lengths + 2·L0)
    int hb_off[FT_MAX_DEPTH];   // hring: first hb row of layer d's slots
    int hb_mask[FT_MAX_DEPTH];  // hring: slot of step t = t & hb_mask[d] (-1: one slot per step)
    long long ncells;    // D*L0*L1
    long long ntiles;    // ncells * naxes * MB * NT
    int dil[FT_MAX_DEPTH];           // KIND_SEQ: per-layer dilation (1 = stacked)
    int ring_off[FT_MAX_DEPTH + 1];  // KIND_SEQ: c-ring slot offset per layer; ring_len = diff
};

struct Cell {
    int k, d, i, j;   // diagonal, depth, position (i = t for KIND_SEQ; j = 0)
    int d0, kl;       // KIND_SEQ: first layer of the cell's band, band-local diagonal
};

FT_HD int num_diagonals(const Problem& p) {
    return p.kind == KIND_SEQ ? p.D + p.L0 - 1 : p.D + p.L0 + p.L1 - 2;
}

FT_HD int imax(int a, int b) { return a > b ? a : b; }
FT_HD int imin(int a, int b) { return a < b ? a : b; }

// First cell (k = 0): (0, 0, 0, 0).
FT_HD Cell first_cell() { return Cell{0, 0, 0, 0, 0, 0}; }

// Successor of `c` in wavefront order: diagonal ascending; within a diagonal depth ascending,
// then i ascending.  For KIND_SEQ the cells of diagonal k are d ∈ [max(0, k-L+1), min(k, D-1)]
// with t = k - d — exactly Table 5's bounds (L355–L358) extended to the boundary regions.
//
// KIND_SEQ generalisation (band, skew): the layers are cut into bands of `band` consecutive
// layers [d0, d0 + nb); band after band, each band runs the hyperplane π = t + skew·(d − d0)
// (a legal schedule for any skew ≥ 1: both dependence vectors e_depth and s·e_time of Table 4
// get π-distance ≥ 1, and every cell of an earlier band precedes the band).  band = D, skew = 1
// is the paper's π = d + t.  A band's weights are what one diagonal reads, so a band that fits in
// L2 turns the per-diagonal weight stream from HBM into L2 hits; skew 2 makes the layer-input
// half of a cell's K loop ready one diagonal before its recurrent half.  Cell.k numbers the
// diagonals globally (bands consecutively).
FT_HD int seq_band(const Problem& p) { return p.band > 0 && p.band < p.D ? p.band : p.D; }
FT_HD int seq_skew(const Problem& p) { return p.skew > 1 ? p.skew : 1; }
FT_HD Cell next_cell(const Problem& p, Cell c) {
    if (p.kind == KIND_SEQ) {
        // no integer division on this path (every role of the kernels walks it per tile): the
        // band start d0 and the band-local diagonal kl are carried in the cell
        const int nbw = seq_band(p), s = seq_skew(p);
        int nb = imin(nbw, p.D - c.d0);
        // next depth on the same diagonal
        if (c.d + 1 < c.d0 + nb && c.kl - s * (c.d + 1 - c.d0) >= 0) {
            c.d += 1;
            c.i = c.kl - s * (c.d - c.d0);
            return c;
        }
        // next non-empty diagonal (of this band, else of the next band)
        for (;;) {
            c.k += 1;
            c.kl += 1;
            if (c.kl > p.L0 - 1 + s * (nb - 1)) {
                c.d0 += nb;
                if (c.d0 >= p.D) {  // past the end: never dereferenced by callers
                    c.d = p.D;
                    c.i = 0;
                    return c;
                }
                nb = imin(nbw, p.D - c.d0);
                c.kl = 0;
            }
            // smallest e = d - d0 with t = kl - s·e <= L0 - 1
            const int over = c.kl - (p.L0 - 1);
            const int e = over > 0 ? (s == 1 ? over : (over + s - 1) / s) : 0;
            if (e <= nb - 1 && c.kl - s * e >= 0) {
                c.d = c.d0 + e;
                c.i = c.kl - s * e;
                c.j = 0;
                return c;
            }
        }
    }
    if (p.band > 0 && p.band < p.D) {
        // KIND_GRID in depth bands: band after band, each a wavefront over kl = i + j + (d − d0)
        // (all three dependence vectors e_depth, e_x, e_y of Table 4 keep kl-distance 1)
        const int nbw = seq_band(p), R = (p.L0 - 1) + (p.L1 - 1);
        int nb = imin(nbw, p.D - c.d0);
        const int r = c.kl - (c.d - c.d0);
        if (c.i < imin(r, p.L0 - 1)) {
            c.i += 1;
            c.j = r - c.i;
            return c;
        }
        for (;;) {
            if (c.d + 1 < c.d0 + nb && c.kl - (c.d + 1 - c.d0) >= 0) {
                c.d += 1;
            } else {
                c.kl += 1;
                c.k += 1;
                if (c.kl > R + nb - 1) {
                    c.d0 += nb;
                    if (c.d0 >= p.D) {  // past the end: never dereferenced by callers
                        c.d = p.D;
                        c.i = c.j = 0;
                        return c;
                    }
                    nb = imin(nbw, p.D - c.d0);
                    c.kl = 0;
                }
                c.d = c.d0 + imax(0, c.kl - R);
            }
            const int rr = c.kl - (c.d - c.d0);
            const int ilo = imax(0, rr - (p.L1 - 1));
            const int ihi = imin(rr, p.L0 - 1);
            if (ilo <= ihi) {
                c.i = ilo;
                c.j = rr - ilo;
                return c;
            }
        }
    }
    // KIND_GRID: diagonal k = d + i + j.
    const int r = c.k - c.d;
    if (c.i < imin(r, p.L0 - 1)) {
        c.i += 1;
        c.j = r - c.i;
        return c;
    }
    for (;;) {
        if (c.d < imin(c.k, p.D - 1)) {
            c.d += 1;
        } else {
            c.k += 1;
            c.d = imax(0, c.k - (p.L0 - 1) - (p.L1 - 1));
        }
        const int rr = c.k - c.d;
        const int ilo = imax(0, rr - (p.L1 - 1));
        const int ihi = imin(rr, p.L0 - 1);
        if (ilo <= ihi) {
            c.i = ilo;
            c.j = rr - ilo;
            return c;
        }
    }
}

// Linear cell index used for flags: KIND_SEQ d*L0 + t, KIND_GRID (d*L0 + i)*L1 + j.
FT_HD long long cell_lin(const Problem& p, int d, int i, int j) {
    return ((long long)d * p.L0 + i) * p.L1 + j;
}

FT_HD int tiles_per_cell(const Problem& p) { return p.naxes * p.MB * p.NT; }

// Flags: one int per (cell, m-block); complete when it reaches naxes * NT * flag_mult
// (cell-granular protocol of the fp32 kernel).
FT_HD int flag_target(const Problem& p) { return p.naxes * p.NT * p.flag_mult; }
// N-tiles of layer 0 (owner mode 3 may run layer 0 in narrower slabs) and the readiness target
// of a cell of layer d (every epilogue warp of every tile of the cell releases once)
FT_HD int nt_layer0(const Problem& p) { return p.nt0 > 0 ? p.nt0 : p.NT; }
FT_HD int flag_target_layer(const Problem& p, int d) {
    return d == 0 ? p.naxes * nt_layer0(p) * p.flag_mult : flag_target(p);
}

// Under layer bands the bf16 streaming kernel publishes a cell twice: the h-ready counter
// flags + cell·MB + m (what the next cells' MMAs read: released as soon as h is stored) and the
// c-ready counter cflag_index() (the cell state, read only by the c-consumer's epilogue: released
// after the c stores, off the h → MMA → h chain).  Both complete at flag_target().  Otherwise
// the h-ready counter covers both.
FT_HD long long cflag_index(const Problem& p, long long cell, int m) {
    return (p.ncells + cell) * p.MB + m;
}

// Monotone cursor over the tile sequence (tile = cell_ordinal * tiles_per_cell + w).  Every
// role of the persistent kernels decodes each of its tiles, so decoding avoids integer division:
// the cursor carries the first tile of its cell and steps cell by cell.
struct Cursor {
    long long ord;    // ordinal of `cell` in wavefront order
    long long tile0;  // = ord * tiles_per_cell
    Cell cell;
};

FT_HD Cursor cursor_begin() { return Cursor{0, 0, first_cell()}; }

FT_HD void cursor_seek(const Problem& p, Cursor& cur, long long target_ord) {
    const int tpc = p.naxes * p.MB * p.NT;
    while (cur.ord < target_ord) {
        cur.cell = next_cell(p, cur.cell);
        ++cur.ord;
        cur.tile0 += tpc;
    }
}

// Decomposition of the within-cell index w = (axis * MB + m) * NT + n.
struct TileId {
    Cell cell;
    int axis, m, n;
};

FT_HD TileId decode_tile(const Problem& p, Cursor& cur, long long tile) {
    const int tpc = tiles_per_cell(p);
    while (tile >= cur.tile0 + tpc) {
        cur.cell = next_cell(p, cur.cell);
        ++cur.ord;
        cur.tile0 += tpc;
    }
    int w = (int)(tile - cur.tile0);
    TileId t;
    t.cell = cur.cell;
    t.axis = 0;
    t.m = 0;
    if (p.naxes == 1 && p.MB == 1) {  // the common case: the within-cell index is the N-tile
        t.n = w;
        return t;
    }
    t.n = w % p.NT;
    w /= p.NT;
    t.m = w % p.MB;
    t.axis = w / p.MB;
    return t;
}

// The tiles one worker (a CTA or a CTA pair) of a persistent kernel processes, in order.
//  * round-robin (default): tiles w, w + nw, w + 2nw, ... of the global wavefront sequence;
//  * owner-computes (p.owner, stacked LSTM under layer bands, one m-block): worker w < band·NT
//    owns the slab (band-local layer e = w / NT, N-tile n = w % NT) and runs it for t = 0 .. T−1
//    in every band (layer d0 + e).  The pair that reads a weight slab is then the same for the
//    whole band (one die's L2 caches it) and the cell state of the slab never leaves the
//    epilogue's registers.  Each worker's sequence follows the dependence order (band, then t),
//    and every dependence (Table 4) points to an earlier (band, t) of another worker or to the
//    worker's own previous tile, so co-resident workers cannot deadlock.
// `tid` identifies the tile for tracing: the global sequence index (round-robin) or
// cell_lin·NT + n (owner).
//  * every layer owned (p.owner == 3, dilated nests with D·NT <= workers): worker w owns
//    (layer w / NT, N-tile w % NT) for t = 0 .. T−1.  Layer e's tile t needs (e − 1, t) of
//    another worker and (e, t − s_e) of its own earlier tiles, and layer 0 depends only on its own
//    steps, so the waits form no cycle.  Each layer then advances at the pace of the layer below
//    with a constant lag instead of queueing behind other layers' tiles.  The cell state stays
//    in registers for layers of dilation 1; the others keep the c ring.
//  * layer-0 owners (p.owner == 2, dilated nests whose layer 0 has dilation 1: its T-step
//    recurrence is the only chain without slack): worker w < NT owns (layer 0, N-tile w) for
//    t = 0 .. T−1, with its cell state in registers; the other workers take the remaining
//    tiles round-robin in wavefront order (a subsequence of the paper order, so the argument
//    above still holds: every dependence points to an earlier tile of the same worker, to a
//    layer-0 owner, which depends on nothing but its own previous steps, or to an earlier tile
//    of the global order).
struct TileWalk {
    Cursor cur;
    long long tile, stride;
    int e, n, d0, t;     // owner modes (e < 0: idle worker; e == -2: round-robin rest)
    long long next, idx0;  // p.owner == 2, the rest: next tile index of this worker among the
                           // non-layer-0 tiles, and that index of the current cell's first tile
};

FT_HD TileWalk walk_begin(const Problem& p, int worker, int nworkers) {
    TileWalk w;
    w.cur = cursor_begin();
    w.tile = worker;
    w.stride = nworkers;
    w.e = -1;
    w.n = 0;
    w.d0 = 0;
    w.t = 0;
    w.next = 0;
    w.idx0 = 0;
    if (p.owner == 1 && worker < seq_band(p) * p.NT) {
        w.e = worker / p.NT;
        w.n = worker - w.e * p.NT;
    } else if (p.owner == 3) {
        const int nt0 = nt_layer0(p);
        if (worker < nt0) {
            w.e = 0;
            w.n = worker;
        } else if (worker - nt0 < (p.D - 1) * p.NT) {
            w.e = 1 + (worker - nt0) / p.NT;
            w.n = (worker - nt0) - (w.e - 1) * p.NT;
        }
    } else if (p.owner == 2) {
        if (worker < p.NT) {
            w.e = 0;
            w.n = worker;
        } else {
            w.e = -2;
            w.next = worker - p.NT;
            w.stride = nworkers - p.NT;
        }
    }
    return w;
}

FT_HD bool walk_next(const Problem& p, TileWalk& w, TileId& tl, long long& tid) {
    if (!p.owner) {
        if (w.tile >= p.ntiles) return false;
        tl = decode_tile(p, w.cur, w.tile);
        tid = w.tile;
        w.tile += w.stride;
        return true;
    }
    if (p.owner == 3) {  // every layer owned: worker (layer e, N-tile n) runs t = 0 .. T-1
        if (w.e < 0 || w.t >= p.L0) return false;
        tl.cell = Cell{w.e + w.t, w.e, w.t, 0, 0, w.e + w.t};
        tl.axis = 0;
        tl.m = 0;
        tl.n = w.n;
        tid = cell_lin(p, w.e, w.t, 0) * (p.nt0 > p.NT ? p.nt0 : p.NT) + w.n;
        ++w.t;
        return true;
    }
    if (p.owner == 2 && w.e == -2) {  // round-robin over the tiles of layers >= 1
        const int tpc = tiles_per_cell(p);
        while (w.cur.ord < p.ncells) {
            if (w.cur.cell.d != 0) {
                if (w.next < w.idx0 + tpc) {
                    tl.cell = w.cur.cell;
                    tl.axis = 0;
                    tl.m = 0;
                    tl.n = (int)(w.next - w.idx0);
                    tid = w.cur.tile0 + tl.n;
                    w.next += w.stride;
                    return true;
                }
                w.idx0 += tpc;
            }
            w.cur.cell = next_cell(p, w.cur.cell);
            ++w.cur.ord;
            w.cur.tile0 += tpc;
        }
        return false;
    }
    if (p.owner == 2) {  // layer-0 owner
        if (w.e != 0 || w.t >= p.L0) return false;
        tl.cell = Cell{w.t, 0, w.t, 0, 0, w.t};
        tl.axis = 0;
        tl.m = 0;
        tl.n = w.n;
        tid = p.ncells * p.NT + (long long)w.t * p.NT + w.n;  // (trace ids past the other tiles')
        ++w.t;
        return true;
    }
    if (w.e < 0) return false;
    const int nbw = seq_band(p);
    while (w.d0 < p.D && w.e >= imin(nbw, p.D - w.d0)) {  // a short last band without layer e
        w.d0 += nbw;
        w.t = 0;
    }
    if (w.d0 >= p.D) return false;
    tl.cell.d = w.d0 + w.e;
    tl.cell.i = w.t;
    tl.cell.j = 0;
    tl.cell.d0 = w.d0;
    tl.cell.kl = w.t + seq_skew(p) * w.e;
    tl.cell.k = tl.cell.kl;
    tl.axis = 0;
    tl.m = 0;
    tl.n = w.n;
    tid = cell_lin(p, tl.cell.d, w.t, 0) * p.NT + w.n;
    if (++w.t == p.L0) {
        w.t = 0;
        w.d0 += nbw;
    }
    return true;
}

// Producer cells of (d, i, j) — the dependence vectors of Table 4 (L307–L317):
// KIND_SEQ: e_depth → (d-1, t), s_d·e_time → (d, t - s_d) (strided access, L331).
// KIND_GRID: e_depth, e_x, e_y → (d-1,i,j), (d,i-1,j), (d,i,j-1).
// Fixed slots (out[k] = linear cell index, or -1 when that producer is outside the domain), so
// callers keep them in registers.  Returns the number of valid producers.
FT_HD int producers(const Problem& p, const Cell& c, long long out[3]) {
    out[0] = c.d > 0 ? cell_lin(p, c.d - 1, c.i, c.j) : -1;
    if (p.kind == KIND_SEQ) {
        const int s = p.dil[c.d];
        out[1] = c.i >= s ? cell_lin(p, c.d, c.i - s, 0) : -1;
        out[2] = -1;
    } else {
        out[1] = c.i > 0 ? cell_lin(p, c.d, c.i - 1, c.j) : -1;
        out[2] = c.j > 0 ? cell_lin(p, c.d, c.i, c.j - 1) : -1;
    }
    return (out[0] >= 0) + (out[1] >= 0) + (out[2] >= 0);
}

// ------------------------------------------------------------------------------------------
// Access materialization (§5.3): the access maps of Fig. 4 (e12 o=[0,-1,0],
// e13 o=[0,0,-1], e14 ws[d], e15 the SSA write, L249–L254) become row coordinates into the
// batch-outermost buffers.  An activation "row" is the middle coordinate of the
// (hidden, rows, batch) view of a buffer: x/ys: position; h_all: (d, t) or (d, i, j, axis).
// ------------------------------------------------------------------------------------------
enum Src : int { SRC_X = 0, SRC_YS = 1, SRC_H = 2, SRC_NONE = 3 };
enum WSel : int { W_IN = 0, W_REC = 1 };

struct Segment {
    int src;    // Src
    int row;    // middle coordinate in the source's (H, rows, B) view
    int wsel;   // WSel
    int slice;  // weight slice: d (seq) or d*2+axis (grid)
    int krow0;  // first K row inside the weight slice (grid U: 0 for h^x, H for h^y)
    int scell;  // SRC_H: linear index of the cell that produced these activations
    int saxis;  // SRC_H: its axis (grid), 0 otherwise
};

// rows per batch row of h_all
FT_HD int h_rows(const Problem& p) {
    return p.kind == KIND_SEQ ? p.D * p.L0 : p.D * p.L0 * p.L1 * 2;
}
FT_HD int h_row(const Problem& p, int d, int i, int j, int a) {
    return p.kind == KIND_SEQ ? d * p.L0 + i : ((d * p.L0 + i) * p.L1 + j) * 2 + a;
}
// Row of the blocked SSA buffer hb that holds h(d, i, j, axis).  Without a ring it is the
// logical row h_row().  With p.hring (bf16 streaming stacked / dilated nests) layer d owns
// slots [hb_off[d], hb_off[d] + len) and step t lives in slot t & hb_mask[d]: the SSA node of
// §4.4 (L217) needs each h only until its consumers have read it — (d, t + s_d) through the
// recurrence and (d + 1, t) through the depth edge (Table 4).  The writer of a wrapped slot waits
// for the depth consumer of the slot's previous step (run_epilogue); the recurrent consumer is
// an ancestor of the writer when len is a multiple of 2·s_d.  A band's last layer (read by the
// next band, which runs after it) keeps every step (hb_mask = -1) in one of two alternating
// regions.
FT_HD int hb_slot_row(const Problem& p, int d, int i, int j, int a) {
    if (p.kind == KIND_SEQ && p.hring) return p.hb_off[d] + (i & p.hb_mask[d]);
    return h_row(p, d, i, j, a);
}
// Ring length of a stacked / dilated layer: the smallest power of two >= max(4, 2·s) when s is a
// power of two (then a multiple of 2·s, see hb_slot_row), else no wrap; never more than T.
FT_HD int hb_ring_len(int s, int T) {
    if (s & (s - 1)) return T;
    int r = 4;
    while (r < 2 * s) r <<= 1;
    return r < T ? r : T;
}

// Slot layout of the hb rings for layer bands of width `band` (0 = one band, the paper order):
// layer d gets hb_ring_len(s_d, T) slots at a running offset; a band's last layer (except the
// last band's) instead keeps all T steps in region (band index & 1) after the rings — the next
// band reads it after this band is done, and the band after that writes the same region only
// after the next band's first layer has read it (a chain of depth edges orders them).
inline void hb_layout(Problem& p, int band) {
    int off = 0;
    for (int d = 0; d < p.D; ++d) {
        const int len = hb_ring_len(p.dil[d], p.L0);
        p.hb_off[d] = off;
        p.hb_mask[d] = len < p.L0 ? len - 1 : -1;
        off += len;
    }
    if (band > 0 && band < p.D)
        for (int d = band - 1; d < p.D - 1; d += band) {
            p.hb_off[d] = off + ((d / band) & 1) * p.L0;
            p.hb_mask[d] = -1;
        }
}

// K rows of one U slice: H (seq) or 2H (grid, acting on s = [h^x; h^y]).
FT_HD int u_krows(const Problem& p) { return p.kind == KIND_SEQ ? p.H : 2 * p.H; }

// The A-operand segments of one tile (the vertical merge x@w + h@u of L609 as one K loop), in
// fixed slots: 0 = layer input, 1 = recurrent state (seq) / h^x_{i-1,j} (grid), 2 = h^y_{i,j-1}
// (grid).  A segment whose producer is outside the domain (t < s, i = 0, j = 0) is the zero
// initial state (scanl s0 = 0, L159/L605) and is marked invalid (skipped): that is the paper's
// boundary region split (region_0..3, L243/L256).  Returns the number of valid segments.
FT_HD int segments(const Problem& p, const TileId& tl, Segment seg[3]) {
    const Cell& c = tl.cell;
    if (p.kind == KIND_SEQ) {
        seg[0] = (c.d == 0) ? Segment{SRC_X, c.i, W_IN, 0, 0, -1, 0}
                            : Segment{SRC_H, hb_slot_row(p, c.d - 1, c.i, 0, 0), W_IN, c.d, 0,
                                      (int)cell_lin(p, c.d - 1, c.i, 0), 0};
        const int s = p.dil[c.d];
        const bool rec = c.i >= s && p.cell == CELL_LSTM;  // the linear cell has no h@U term
        seg[1] = Segment{rec ? SRC_H : SRC_NONE, rec ? hb_slot_row(p, c.d, c.i - s, 0, 0) : 0,
                         W_REC, c.d, 0, rec ? (int)cell_lin(p, c.d, c.i - s, 0) : -1, 0};
        seg[2] = Segment{SRC_NONE, 0, W_REC, c.d, 0, -1, 0};
        // Dilation s >= 2: the recurrent producer (d, t − s) lies s − 1 diagonals before the
        // depth producer (d − 1, t), so it is (almost always) ready first.  Running its half of
        // the K loop first leaves only the depth half behind the depth edge, which cuts the
        // latency of every layer-to-layer hop of a dilated nest by one half-K of MMAs.  The sum
        // is the same (the K halves are added in a different order: equal within rounding).
        if (p.rec_first && rec && s >= 2 && c.d > 0) {
            const Segment t0 = seg[0];
            seg[0] = seg[1];
            seg[1] = t0;
        }
    } else {
        const int a = tl.axis, sl = c.d * 2 + a;
        if (c.d == 0)
            seg[0] = Segment{a == 0 ? SRC_X : SRC_YS, a == 0 ? c.i : c.j, W_IN, sl, 0, -1, 0};
        else
            seg[0] = Segment{SRC_H, h_row(p, c.d - 1, c.i, c.j, a), W_IN, sl, 0,
                             (int)cell_lin(p, c.d - 1, c.i, c.j), a};
        seg[1] = Segment{c.i > 0 ? SRC_H : SRC_NONE, c.i > 0 ? h_row(p, c.d, c.i - 1, c.j, 0) : 0,
                         W_REC, sl, 0, c.i > 0 ? (int)cell_lin(p, c.d, c.i - 1, c.j) : -1, 0};
        seg[2] = Segment{c.j > 0 ? SRC_H : SRC_NONE, c.j > 0 ? h_row(p, c.d, c.i, c.j - 1, 1) : 0,
                         W_REC, sl, p.H, c.j > 0 ? (int)cell_lin(p, c.d, c.i, c.j - 1) : -1, 1};
    }
    return 1 + (seg[1].src != SRC_NONE) + (seg[2].src != SRC_NONE);
}

// Index of the next valid segment after slot `si` (3 when none is left).
FT_HD int next_segment(const Segment seg[3], int si) {
    if (si < 1 && seg[1].src != SRC_NONE) return 1;
    if (si < 2 && seg[2].src != SRC_NONE) return 2;
    return 3;
}

// rows per batch row of each activation source
FT_HD int src_rows(const Problem& p, int src) {
    return src == SRC_X ? p.L0 : (src == SRC_YS ? p.L1 : h_rows(p));
}

// Cell-state ring (fp32).  KIND_SEQ: layer d owns ring_len_d = min(T, s_d) slots
// [ring_off[d], ring_off[d+1]); slot of step t is t mod ring_len_d.  The slot cell (d, t) writes
// held c(d, t - s_d), which only (d, t) itself reads — the same threads, the same elements, read
// before they are overwritten — and the next writer (d, t + s_d) depends on (d, t), so the reuse
// is ordered by the flag protocol.  (Round 1 kept 2·s_d slots per layer.)  KIND_GRID: ONE c^x slot per (depth, column j) and one
// c^y slot per (depth, row i) ([D][Ly] + [D][Lx] slots): c^x(d, i−1, j) is read only by cell
// (d, i, j) — the same threads that then overwrite the same elements with c^x(d, i, j) — and the
// next writer (d, i+1, j) depends on (d, i, j) (e_x of Table 4), so one slot carries the chain.
// (Round 1 kept 2 slots: 32 MiB of rings per C5 depth instead of 16.)
// Inside a slot the layout is [H/4][B][4]: 4 units of one batch row are one 16-byte vector and
// consecutive batch rows are adjacent, so an epilogue warp (one thread per batch row) loads and
// stores whole 512-byte runs.  (A [B][H] slot made every warp store 32 partial sectors 4 KiB
// apart; those stores cost 23 % of C3's energy at the power cap — profiles/r2_power.)
FT_HD long long c_slot_elems(const Problem& p) { return (long long)((p.H + 3) >> 2) * 4 * p.B; }
FT_HD long long c_slot_index(const Problem& p, long long slot, int b, int n) {
    return ((slot * ((p.H + 3) >> 2) + (n >> 2)) * p.B + b) * 4 + (n & 3);
}
FT_HD long long c_ring_index(const Problem& p, int d, int i, int j, int a, int b, int n) {
    if (p.kind == KIND_SEQ) {
        const int len = p.ring_off[d + 1] - p.ring_off[d];
        return c_slot_index(p, p.ring_off[d] + i % len, b, n);
    }
    if (a == 0) return c_slot_index(p, (long long)d * p.L1 + j, b, n);
    const long long base = (long long)p.D * p.L1;
    return c_slot_index(p, base + (long long)d * p.L0 + i, b, n);
}

// The cell whose c the tile's epilogue reads (its c-producer), or -1 (zero initial state).
FT_HD long long c_producer(const Problem& p, const TileId& tl, int* pi, int* pj) {
    const Cell& c = tl.cell;
    if (p.kind == KIND_SEQ) {
        const int s = p.dil[c.d];
        if (c.i < s) return -1;
        *pi = c.i - s;
        *pj = 0;
        return cell_lin(p, c.d, c.i - s, 0);
    }
    if (tl.axis == 0) {
        if (c.i == 0) return -1;
        *pi = c.i - 1;
        *pj = c.j;
        return cell_lin(p, c.d, c.i - 1, c.j);
    }
    if (c.j == 0) return -1;
    *pi = c.i;
    *pj = c.j - 1;
    return cell_lin(p, c.d, c.i, c.j - 1);
}

// bf16 path: the SSA activations live in a blocked, batch-contiguous layout
//   hb[row][kc][Bp][64]   (row = h_row(), kc = unit / 64, Bp = MB * BM batch rows incl. padding)
// so that the A operand of one tile K-chunk (128 batch rows x 64 units) is one contiguous 16 KiB
// block: a 2-D TMA box with no large strides, and the epilogue's h stores are coalesced.
FT_HD long long hb_rows_total(const Problem& p) {
    return (long long)(p.kind == KIND_SEQ && p.hring ? p.hb_rows : h_rows(p)) * (p.H / 64) *
           ((long long)p.MB * p.BM);
}
FT_HD long long hb_row(const Problem& p, int row, int kc, int b) {
    return ((long long)row * (p.H / 64) + kc) * ((long long)p.MB * p.BM) + b;
}

// Output element indices (batch row b, unit n).
FT_HD long long h_all_index(const Problem& p, const Cell& c, int a, int b, int n) {
    return ((long long)b * h_rows(p) + h_row(p, c.d, c.i, c.j, a)) * p.H + n;
}
// y (seq, top layer) / out (grid, top depth); valid only when c.d == D-1.
FT_HD long long y_index(const Problem& p, const Cell& c, int a, int b, int n) {
    if (p.kind == KIND_SEQ) return ((long long)b * p.L0 + c.i) * p.H + n;
    return ((((long long)b * p.L0 + c.i) * p.L1 + c.j) * 2 + a) * (long long)p.H + n;
}
// h_n / c_n; valid only at the last position.
FT_HD bool is_last_pos(const Problem& p, const Cell& c) {
    return p.kind == KIND_SEQ ? c.i == p.L0 - 1 : (c.i == p.L0 - 1 && c.j == p.L1 - 1);
}
FT_HD long long hn_index(const Problem& p, const Cell& c, int a, int b, int n) {
    return ((long long)b * p.D + c.d) * (long long)p.naxes * p.H + (long long)a * p.H + n;
}

}  // namespace ft

#ifdef __CUDACC__
namespace ft {

#ifndef FT_SPIN_TIMEOUT_NS
#define FT_SPIN_TIMEOUT_NS 20000000000ull  // 20 s: a lost dependency traps instead of hanging
#endif

__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ int ld_acquire_gpu(const int* p) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ int ld_relaxed_gpu(const int* p) {
    int v;
    asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// acquire fence: with the relaxed loads before it that observed released values, this gives
// those loads acquire semantics (fence-based synchronization of the PTX memory model)
__device__ __forceinline__ void fence_acq_rel_gpu() {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
}

__device__ __forceinline__ void red_release_gpu_add(int* p, int v) {
    asm volatile("red.release.gpu.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ void fence_acq_rel_sys() {
    asm volatile("fence.acq_rel.sys;" ::: "memory");
}
__device__ __forceinline__ void red_relaxed_sys_add(int* p, int v) {
    asm volatile("red.relaxed.sys.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Bounded acquire-spin (system scope) on a flag written by a copy stream (cuStreamWriteValue32).
__device__ __forceinline__ int ld_acquire_sys(const int* p) {
    int v;
    asm volatile("ld.acquire.sys.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void wait_flag_geq_sys(const int* p, int target) {
    if (ld_acquire_sys(p) >= target) return;
    const uint64_t t0 = globaltimer_ns();
    for (;;) {
        __nanosleep(256);
        if (ld_acquire_sys(p) >= target) return;
        if (globaltimer_ns() - t0 > FT_SPIN_TIMEOUT_NS) __trap();
    }
}

// Bounded acquire-spin on a readiness counter.
__device__ __forceinline__ void wait_flag_geq(const int* p, int target) {
    if (ld_acquire_gpu(p) >= target) return;
    const uint64_t t0 = globaltimer_ns();
    for (;;) {
#ifdef FT_POLL_RELAXED  // experiment: spin on relaxed loads (no L1 invalidate per poll), then
                        // one acquire load of the (monotone) counter once it is there
#pragma unroll 1
        for (int it = 0; it < 256; ++it)
            if (ld_relaxed_gpu(p) >= target) {
                (void)ld_acquire_gpu(p);
                return;
            }
#else
#pragma unroll 1
        for (int it = 0; it < 256; ++it)
            if (ld_acquire_gpu(p) >= target) return;
#endif
        if (globaltimer_ns() - t0 > FT_SPIN_TIMEOUT_NS) __trap();
    }
}

}  // namespace ft
#endif
