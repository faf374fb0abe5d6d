/*
 * ft_oracle.c — CPU ORACLE.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  The product path (paper_conf_sosp_liuqc0hs0y24_b200/) never links,
 * imports or calls it, and this file shares no code, header or constant with the CUDA path.
 *
 * What it computes: the plain definition of the nested recurrence
 *     map(batch) ∘ scan(depth) ∘ scan(time)
 * of FractalTensor (SOSP'24), written as the loop nest of the paper's listings, in the paper's
 * order (batch outermost), with no blocking, fusion or reordering:
 *
 *   stacked LSTM  — Listing 2, PAPER.md L590–L616 (cell L607–L615), scanl semantics Table 1
 *                   L117–L118 (output excludes s0, s0 = (0,0) L605).
 *   dilated RNN   — the same cell; the time scan reads t - s_d (constantly strided access, L134;
 *                   "the dependence distance becomes the stride", L331); dilation range L381.
 *   grid RNN      — three nested scans (depth, x, y): 8 block nodes (L421); cell reading
 *                   DESIGN.md R12–R14 (Grid LSTM [18], L497): per-axis LSTM transforms sharing
 *                   s = [h^x_{i-1,j}; h^y_{i,j-1}].  PARITY UNPINNED BY THE PAPER beyond the
 *                   Ly=1 / Lx=1 reductions (tests P8) — the paper never defines the grid cell.
 *                   The reading itself is pinned by P8/P8b (reductions, axis swap), P8c (no
 *                   recurrence: per-axis batched-matmul closed form) and P8d (dependence cone).
 *
 * Readings of the paper: gate order (i,f,o,ĝ) = gs[0..3] (L611–L615,
 * R1/R2); W multiplies the layer input, U the recurrent h (R3, "x@w + h@u", L609); one bias per
 * gate (R4, L599/L609); row-vector convention z = a·W, W[k][n] (R5, L174); layer d>=1 input is
 * layer d-1's h (R6, Listing 1); zero initial state (R7).
 *
 * Summation order (fixed, documented): z = b, then + a[k]·W[k][n] for k ascending, then
 * + hp[k]·U[k][n] for k ascending.  The k-outer / n-inner loop below performs exactly that
 * sequence of additions for every output (it only changes which output is updated next).
 *
 * Precision: REAL = double (the parity reference) or float (CPU timing instantiation), plus a
 * DIAGNOSTIC-ONLY third build, _bf16emu: float with h rounded to bf16 (round-to-nearest-even)
 * after every cell, mirroring the rounding point of the bf16 GPU path (R20; SURVEY
 * §8(c) c.4).  It separates kernel bugs from precision effects and is never the judged reference.
 * Parallelism: OpenMP over the batch map only (fully parallel, Table 1 map, L126); this does
 * not change any output's arithmetic.
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>

#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_EXPORT __attribute__((visibility("default")))

/* float -> nearest bf16 (ties to even), returned as float; finite inputs only */
static float oracle_round_bf16(float v) {
    unsigned int u;
    memcpy(&u, &v, sizeof(u));
    u += 0x7FFFu + ((u >> 16) & 1u);
    u &= 0xFFFF0000u;
    memcpy(&v, &u, sizeof(v));
    return v;
}

/* ---------------------------------------------------------------------------------------- */
/* instantiate three times: _f64 (parity), _f32 (timing), _bf16emu (diagnostic)             */
/* ---------------------------------------------------------------------------------------- */
#define REAL double
#define SFX(name) name##_f64
#define EXPF exp
#define TANHF tanh
#define ROUND_H(v) (v)
#include "ft_oracle_impl.h"
#undef REAL
#undef SFX
#undef EXPF
#undef TANHF

#define REAL float
#define SFX(name) name##_f32
#define EXPF expf
#define TANHF tanhf
#include "ft_oracle_impl.h"
#undef SFX
#undef ROUND_H

/* diagnostic: float with h rounded to bf16 after every LSTM cell */
#define SFX(name) name##_bf16emu
#define ROUND_H(v) oracle_round_bf16(v)
#include "ft_oracle_impl.h"
#undef REAL
#undef SFX
#undef EXPF
#undef TANHF
#undef ROUND_H

ORACLE_EXPORT int ft_oracle_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

ORACLE_EXPORT int ft_oracle_version(void) { return 1; }
