// wavefront_bf16.cu — BK2/BK3/BK4: the persistent sm_100a wavefront (stacked, dilated, grid).
//
// One launch runs the whole nest.  Every CTA (one per SM; all co-resident) walks the global tile
// sequence in wavefront order (ft_common.cuh).  A tile = (cell, axis, M batch rows, 64 hidden
// units x 4 gates):
//
//   z[M x 256] = Σ_seg A_seg[M x H] · B_seg[H x 256] + b          (Listing 2)
//
// the horizontal merge of the 4 gate maps (N = 4 x 64, L287) and the vertical merge of
// x@w + h@u (K = segments x H, L289–L293) as one tcgen05 GEMM; A = activation rows (batch = the
// GEMM M dimension — the reuse dimension of L345–L349), B = the weight slice W[d][g][k][n] used
// as an MN-major operand (n contiguous, no repacking).  The LSTM update (L611–L615) runs in the
// epilogue straight out of TMEM.
//
// Two instantiations:
//   CG = 1  one CTA per tile, M = 128 (batch <= 128)
//   CG = 2  a CTA pair (cluster of 2, tcgen05 cta_group::2) per tile, M = 256: each CTA stages its
//           128 A rows and HALF of the N = 256 weight columns (gates i,f or o,ĝ); the leader CTA
//           issues M256 N256 K16 MMAs reading both CTAs' shared memory, so each weight tile is
//           fetched once per cell for the whole 256-row batch and per-CTA weight traffic halves.
// Each comes in 64-unit (N = 256) and 32-unit (N = 128) N-tiles.  Dilated nests run one launch
// with two widths (wavefront_bf16_kernel<2, 64, 32>): the CTA pairs that own layer 0 — the only
// recurrence without slack — run 32-unit slabs, every other pair 64-unit slabs (kernel_body per
// CTA; TileWalk owner mode 3 in ft_common.cuh).
//
// Warp roles (352 threads per CTA with the default FT_EPI_WARPS = 8; 16 epilogue warps measured
// slower: C3 6.30 -> 6.61 ms, C4 0.871 -> 0.903 ms, profiles/r2_ab_epi_warps.txt):
//   warp 0      weight TMA producer: streams the 64-deep K-chunks of B (no dependencies) into a
//               STAGES-deep shared-memory ring (mbarriers), running ahead of the wavefront.
//   warp 10     activation TMA producer: waits the tile's producer cells (readiness counters),
//               then streams the matching K-chunks of A into the same ring slots.
//   warp 1      MMA issuer (leader CTA): one thread issues tcgen05.mma into a double-buffered
//               TMEM accumulator (2 x 256 fp32 columns) so tile n+1's MMAs overlap tile n's
//               epilogue.
//   warps 2-9   epilogue (2 warps per TMEM lane quadrant, 32 units each): tcgen05.ld → +b, σ/σ/σ/tanh, c' = f·c + i·ĝ, h' = o·tanh(c') in fp32
//               registers; h' → bf16 → h_all (the SSA buffer node, L217) and y / h_n; c' → fp32
//               cell-state ring (+ c_all / c_n); then release the tile's share of the
//               (cell, m-block) readiness counter.
//
// Cross-CTA ordering (generic-proxy stores → another SM's async-proxy TMA loads):
//   writer: st.global …; bar.sync (epilogue warps); one thread fence.acq_rel.gpu + red.release.gpu
//   reader: ld.acquire.gpu (bounded spin); fence.proxy.async.global; cp.async.bulk.tensor
// L2 policy: streamed weights EVICT_FIRST (they are re-read only one diagonal later, after the
// whole 256 MiB weight set went through L2), weights of the first `resident_layers` layers
// EVICT_LAST (kept in L2 across time steps — the reuse of L345–L349), activations EVICT_NORMAL.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>

#include "ft_internal.h"
#include "ft_sm100.cuh"

namespace ft {

#ifdef FT_TRACE
// Development-only role timing (built into libft_trace.so by tools/trace_build.sh, never into
// libft.so): per CTA, cycles spent in each wait / work phase.
enum TraceSlot {
    TR_P_FLAG = 0, TR_P_EMPTY, TR_M_FULL, TR_M_TEMPTY, TR_E_TFULL, TR_E_WORK, TR_E_CFLAG, TR_TOTAL,
    TR_TILES, TR_E_LDTM, TR_E_MATH, TR_E_STORE, TR_E_BAR, TR_E_REL, TR_SLOTS = 16
};
__device__ unsigned long long g_trace[1024 * TR_SLOTS];
// per-tile event timestamps (%globaltimer, ns) of the leader CTA: 0 wait start, 1 deps ready,
// 2 A loads issued, 3 MMA done (epilogue saw tfull), 4 counter released, 5 last producer flag
// acquired, 6 MMA warp got the accumulator, 7 MMA warp issued the last chunk, 8 A producer got
// the slot of the last segment's first chunk, 9 A producer got the slot of the tile's last
// chunk, 10 MMA saw the last segment's first chunk land, 11 MMA saw the chunk before it land,
// 12 weight producer issued the tile's last weight chunk
constexpr int EV_MAX_TILES = 32768;
constexpr int EV_K = 16;
__device__ unsigned long long g_events[EV_MAX_TILES * EV_K];
#define FT_EV(tile, k) do { if ((tile) < EV_MAX_TILES) g_events[(tile) * EV_K + (k)] = globaltimer_ns(); } while (0)
// register accumulators, flushed once per role (keeps the instrumented loops lean)
#define FT_TR_ROLE unsigned long long _acc[TR_SLOTS] = {0}
#define FT_TR_DECL long long _tr0 = 0
#define FT_TR_BEGIN() (_tr0 = clock64())
#define FT_TR_END(slot) (_acc[(slot)] += (unsigned long long)(clock64() - _tr0))
#define FT_TR_ADD(slot, v) (_acc[(slot)] += (unsigned long long)(v))
#define FT_TR_FLUSH(cond)                                                          \
    do {                                                                           \
        if (cond)                                                                  \
            for (int _k = 0; _k < TR_SLOTS; ++_k)                                  \
                if (_acc[_k]) g_trace[blockIdx.x * TR_SLOTS + _k] += _acc[_k];     \
    } while (0)
#else
#define FT_TR_ROLE
#define FT_TR_DECL
#define FT_TR_BEGIN() ((void)0)
#define FT_TR_END(slot) ((void)0)
#define FT_TR_ADD(slot, v) ((void)0)
#define FT_TR_FLUSH(cond) ((void)0)
#ifdef FT_TRACE_LIGHT  // development (tools/c4_spread.py): events 1-5, 7-11 only, no role
                       // counters — close to the release build's timing
constexpr int EV_MAX_TILES = 32768;
constexpr int EV_K = 16;
__device__ unsigned long long g_events[EV_MAX_TILES * EV_K];
#define FT_EV(tile, k) do { if ((k) != 0 && (k) != 6 && (k) != 12 && (tile) < EV_MAX_TILES) g_events[(tile) * EV_K + (k)] = globaltimer_ns(); } while (0)
// (13 first TMEM chunk in the epilogue's registers, 14 math and h stores issued: light build only)
#else
#define FT_EV(tile, k) ((void)0)
#endif
#endif

namespace {

using namespace sm100;

constexpr int ROWS = BF16_BM;  // 128 batch rows per CTA = TMEM lanes
constexpr int BK = 64;         // K per stage = one 128-byte swizzle row of bf16 (A operand)
constexpr int UK = 16;         // UMMA K for kind::f16
// Epilogue warps: 4 TMEM lane quadrants x EPI_PARTS unit ranges of the tile.
#ifndef FT_EPI_WARPS
#define FT_EPI_WARPS 8
#endif
constexpr int EPI_WARPS = FT_EPI_WARPS;
constexpr int EPI_PARTS = EPI_WARPS / 4;
constexpr int EPI_THREADS = EPI_WARPS * 32;
constexpr int ACT_WARP = 2 + EPI_WARPS;   // the activation TMA producer
// warp 0 weight TMA, 1 MMA, 2 .. 1+EPI_WARPS epilogue, ACT_WARP activation TMA
constexpr int THREADS = 32 * (3 + EPI_WARPS);

// Tile configuration: CG CTAs per tile (1 or a cta_group::2 pair), U hidden units per N-tile
// (64: N = 256 with 128-byte-swizzled weight atoms; 32: N = 128 with 64-byte swizzle — twice the
// tiles per diagonal at half the per-tile latency, for diagonals too narrow to fill the GPU).
template <int CG, int U>
struct KCfg {
    static constexpr int BN = 4 * U;                           // UMMA N (i | f | o | ĝ)
    static constexpr int TMEM_COLS = 2 * BN;                   // double-buffered accumulator
    static constexpr int GATES = 4 / CG;                       // weight gate atoms per CTA
    static constexpr int WROW = U * 2;                         // bytes per weight smem row
    static constexpr uint32_t WLAYOUT = U == 64 ? 2u : 4u;     // SWIZZLE_128B / SWIZZLE_64B
    static constexpr int A_BYTES = ROWS * BK * 2;              // 16 KiB
    static constexpr int B_BYTES = GATES * U * BK * 2;         // weight atoms of one K chunk
    static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
    static constexpr int STAGES = (196 * 1024) / STAGE_BYTES;  // 4 / 6 / 6 / 8
    static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 256 + 2048 /* bias x 2 */ + 1024 /* align */;
    static constexpr uint32_t IDESC = make_idesc_bf16_f32(ROWS * CG, BN, false, true);
    static constexpr int EPI_UNITS = U / EPI_PARTS;            // units per epilogue thread
    // units per TMEM load: 16, or 8 with 16 epilogue warps (register budget of 608 threads)
#ifdef FT_EPI_CH  // experiments: 8 or 16
    static constexpr int EPI_CH = EPI_UNITS < FT_EPI_CH ? EPI_UNITS : FT_EPI_CH;
#else
    static constexpr int EPI_CH = EPI_UNITS < 16 / EPI_PARTS * 2 ? EPI_UNITS : 16 / EPI_PARTS * 2;
#endif
};

struct Maps {
    CUtensorMap x, ys, h, W, U;
    CUtensorMap xd;  // x [B][T][H] as (H, T, B), box (64, 1, 128): layer-0 inputs when P.x_direct
};

__device__ __forceinline__ int weight_layer(const Problem& P, int slice) {
    return P.kind == KIND_SEQ ? slice : slice >> 1;
}

// L2 eviction policy from a 2-bit override code (0 = keep `dflt`).
__device__ __forceinline__ uint64_t l2_policy(int code, uint64_t dflt) {
    return code == 1 ? policy_evict_first() : code == 2 ? policy_evict_normal()
                                             : code == 3 ? policy_evict_last() : dflt;
}

// ------------------------------------------------------------------------------ producer
// The weight (B) half of a stage does not depend on any other cell, only the activation (A) half
// does.  So for each tile the producer first claims up to STAGES ring slots and starts their
// weight loads (the HBM stream), THEN waits for the producer cells' readiness counters, then
// issues the activation loads of those slots: the weight latency hides behind the dependency wait.
// The loop is kept lean (no division, no local-memory arrays, precomputed shared addresses): one
// thread must issue a 32–48 KiB stage every ~512 tensor cycles.
__device__ __forceinline__ Segment pick(const Segment (&seg)[3], int i) {
    Segment r;  // field-wise selects keep the three segments in registers
    r.src = i == 0 ? seg[0].src : (i == 1 ? seg[1].src : seg[2].src);
    r.row = i == 0 ? seg[0].row : (i == 1 ? seg[1].row : seg[2].row);
    r.wsel = i == 0 ? seg[0].wsel : (i == 1 ? seg[1].wsel : seg[2].wsel);
    r.slice = i == 0 ? seg[0].slice : (i == 1 ? seg[1].slice : seg[2].slice);
    r.krow0 = i == 0 ? seg[0].krow0 : (i == 1 ? seg[1].krow0 : seg[2].krow0);
    r.scell = i == 0 ? seg[0].scell : (i == 1 ? seg[1].scell : seg[2].scell);
    r.saxis = i == 0 ? seg[0].saxis : (i == 1 ? seg[1].saxis : seg[2].saxis);
    return r;
}

// A operand K-chunk kc of segment sg for batch rows arow0 .. arow0+127, always from a blocked
// [row][kc][Bp][64] buffer (2-D TMA, one contiguous 16 KiB box): the SSA activations hb, or the
// layer-0 inputs x / ys packed into that layout at the start of the call (pack_rows_kernel).
template <int CG>
__device__ __forceinline__ void load_a(const Problem& P, const Maps& M, uint32_t dst, uint32_t bar,
                                       const Segment& sg, int kc, int arow0, bool fixed, uint64_t pol) {
    if (sg.src == SRC_X && P.x_direct && !fixed) {  // straight from x [B][T][H] (no pack)
        tma_load_3d_hint_addr<CG>(dst, &M.xd, bar, kc * BK, sg.row, arow0, pol);
        return;
    }
    const CUtensorMap* am = (fixed || sg.src == SRC_X) ? &M.x : (sg.src == SRC_YS ? &M.ys : &M.h);
    tma_load_2d_hint_addr<CG>(dst, am, bar, 0, fixed ? arow0 : (int)hb_row(P, sg.row, kc, arow0), pol);
}

// Pack a caller input [B][L][H] (batch-outermost, the ABI layout) into the blocked layout
// [L][H/64][Bp][64] the A-operand boxes read; rows B..Bp-1 are zero.  One 16-byte vector per
// thread-iteration, coalesced on the write side.
__global__ void pack_rows_kernel(const __nv_bfloat16* __restrict__ src, __nv_bfloat16* __restrict__ dst,
                                 int B, int L, int H, int Bp) {
    const int KC = H / 64;
    const long long nvec = (long long)L * KC * Bp * 8;
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nvec;
         v += (long long)gridDim.x * blockDim.x) {
        const int j = (int)(v & 7);
        long long r = v >> 3;
        const int b = (int)(r % Bp);
        r /= Bp;
        const int kc = (int)(r % KC);
        const int l = (int)(r / KC);
        uint4 val = make_uint4(0, 0, 0, 0);
        if (b < B)
            val = __ldg(reinterpret_cast<const uint4*>(src + ((long long)b * L + l) * H + kc * 64 + j * 8));
        reinterpret_cast<uint4*>(dst)[v] = val;
    }
}

// Two producer threads in different warps share the ring: the WEIGHT producer (no dependencies,
// runs up to STAGES chunks ahead, i.e. the HBM weight stream never waits for the wavefront) and
// the ACTIVATION producer (acquires the tile's producer cells, then loads A).  Each ring slot's
// full barrier (in the leader CTA) takes one expect-tx arrival from each of the leader's two
// producers; the peer CTA's producers only issue loads.  Splitting halves the serial TMA issue
// work per thread (the role trace showed one thread issuing both was the limiter).
template <int CG, int U, bool kWeights>
__device__ __forceinline__ void run_producer(const Problem& P, const Tensors& T, const Maps& M,
                                             uint8_t* sA, uint8_t* sB, uint64_t* full,
                                             uint64_t* empty, uint32_t rank) {
    using C = KCfg<CG, U>;
    const uint32_t sA0 = smem_u32(sA), sB0 = smem_u32(sB);
    const uint32_t full0 = (CG == 2) ? mapa_shared(smem_u32(full), 0) : smem_u32(full);
    int stage = 0;
    uint32_t phase = 0;
    const int target = flag_target(P), target0 = flag_target_layer(P, 0);
    const long long l0cells = (long long)P.L0 * P.L1;  // cells of layer 0 come first (cell_lin)
    const int kchunks = P.H / BK;
    uint64_t pol_stream = policy_evict_first();
    uint64_t pol_keep = policy_evict_last();
    const uint64_t pol_act = l2_policy((P.l2pol >> 4) & 3, policy_evict_normal());
    if (P.l2pol & 3) pol_stream = pol_keep = l2_policy(P.l2pol & 3, pol_keep);
    const bool skipB = FT_DEV_BIT(P.debug, 16), fixed = FT_DEV_BIT(P.debug, 32);  // timing experiments
    const uint32_t tx = kWeights ? (skipB ? 0 : CG * C::B_BYTES) : CG * C::A_BYTES;
    TileWalk walk = walk_begin(P, blockIdx.x / CG, gridDim.x / CG);
    FT_TR_ROLE;
    TileId tl;
    long long tile;
    while (walk_next(P, walk, tl, tile)) {
        Segment seg[3];
        const int ns = segments(P, tl, seg);
        const int nchunks = ns * kchunks;
        const int arow0 = tl.m * ROWS * CG + (int)rank * ROWS;
        const bool lin = P.cell == CELL_LINEAR;
        const int bn = (fixed || lin) ? 0 : tl.n * U;
        const int bg = (lin ? tl.n * 4 : 0) + (int)rank * C::GATES;
        FT_TR_DECL;
        if constexpr (!kWeights) {
            FT_TR_ADD(TR_TILES, 1);
            if (rank == 0) FT_EV(tile, 0);
        }
        int si = 0, kc = 0;
        for (int c = 0; c < nchunks; ++c) {
            const Segment sg = pick(seg, si);
            if constexpr (!kWeights) {
                // the segment's producer cell (Table 4 dependence vectors): one acquire of its
                // (cell, m-block) counter before the segment's first activation load, so inputs
                // that are ready (x, the layer below) stream in while a later producer finishes
                if (kc == 0 && sg.scell >= 0 && !FT_DEV_BIT(P.debug, 1)) {
                    FT_TR_BEGIN();
                    wait_flag_geq(T.flags + (long long)sg.scell * P.MB + tl.m, sg.scell < l0cells ? target0 : target);
                    FT_TR_END(TR_P_FLAG);
                    if (rank == 0) FT_EV(tile, 5);
                    fence_proxy_async_global();
                }
                if (kc == 0 && sg.src == SRC_X && T.xsig) {  // host-IO: this x chunk has landed
                    wait_flag_geq_sys(T.xsig + sg.row / T.xchunk, 1);
                    fence_proxy_async_global();
                }
                if (c == 0 && rank == 0) FT_EV(tile, 1);
            }
            if constexpr (kWeights) FT_TR_BEGIN();
            mbar_wait(&empty[stage], phase ^ 1);
            if constexpr (kWeights) FT_TR_END(TR_P_EMPTY);
#if defined(FT_TRACE) || defined(FT_TRACE_LIGHT)
            if constexpr (!kWeights) {
                if (rank == 0 && c == nchunks - kchunks) FT_EV(tile, 8);
                if (rank == 0 && c == nchunks - 1) FT_EV(tile, 9);
            }
#endif
            const uint32_t bar = full0 + 8u * (uint32_t)stage;
            if (rank == 0) mbar_arrive_expect_tx(&full[stage], tx);
            if constexpr (kWeights) {
                if (!skipB) {
                    const CUtensorMap* bm = sg.wsel == W_IN ? &M.W : &M.U;
                    const int wl = weight_layer(P, sg.slice);
                    const uint64_t wpol = (sg.wsel == W_IN && wl < P.persist_layers)
                                              ? pol_act
                                              : (wl < P.resident_layers ? pol_keep : pol_stream);
                    tma_load_4d_hint_addr<CG>(sB0 + (uint32_t)(stage * C::B_BYTES), bm, bar, bn,
                                              fixed ? 0 : sg.krow0 + kc * BK, bg, fixed ? 0 : sg.slice, wpol);
                }
            } else {
                load_a<CG>(P, M, sA0 + (uint32_t)(stage * C::A_BYTES), bar, sg, kc, arow0, fixed, pol_act);
            }
            if (++kc == kchunks) { kc = 0; si = next_segment(seg, si); }
            if (++stage == C::STAGES) {
                stage = 0;
                phase ^= 1;
            }
        }
        if constexpr (!kWeights) if (rank == 0) FT_EV(tile, 2);
        if constexpr (kWeights) if (rank == 0) FT_EV(tile, 12);
    }
    FT_TR_FLUSH(true);  // the two producers fill disjoint slots
}

// ------------------------------------------------------------------------------ MMA issuer
template <int CG, int U>
__device__ __forceinline__ void run_mma(const Problem& P, uint32_t tmem_base, uint8_t* sA,
                                        uint8_t* sB, uint64_t* full, uint64_t* empty,
                                        uint64_t* tfull, uint64_t* tempty) {
    using C = KCfg<CG, U>;
    int stage = 0;
    uint32_t phase = 0;
    int acc = 0;
    uint32_t acc_phase = 0;
    const int kchunks = P.H / BK;
    // A: K-major, SW128: 128-B rows, 8-row groups 1024 B apart (SBO); K step = +32 B.
    // B: MN-major, U-unit swizzle atoms (one per gate) U*64*2 B apart (LBO), 8-k-row groups
    //    8*WROW apart (SBO); K step of 16 rows = 16*WROW.  CG 2: each CTA holds half the atoms.
    const uint64_t adesc0 = make_sdesc(smem_u32(sA), 16, 1024);
    const uint64_t bdesc0 = make_sdesc(smem_u32(sB), U * BK * 2, 8 * C::WROW, C::WLAYOUT);
    TileWalk walk = walk_begin(P, blockIdx.x / CG, gridDim.x / CG);
    FT_TR_ROLE;
    TileId tl;
    long long tile;
    while (walk_next(P, walk, tl, tile)) {
        Segment seg[3];
        const int nchunks = segments(P, tl, seg) * kchunks;
        FT_TR_DECL;
        FT_TR_BEGIN();
        mbar_wait_warp(&tempty[acc], acc_phase ^ 1);
        FT_TR_END(TR_M_TEMPTY);
        if ((threadIdx.x & 31) == 0) FT_EV(tile, 6);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + (uint32_t)(acc * C::BN);
        for (int c = 0; c < nchunks; ++c) {
            FT_TR_BEGIN();
            mbar_wait_warp(&full[stage], phase);
            FT_TR_END(TR_M_FULL);
#if defined(FT_TRACE) || defined(FT_TRACE_LIGHT)
            if ((threadIdx.x & 31) == 0 && c == nchunks - kchunks) FT_EV(tile, 10);
            if ((threadIdx.x & 31) == 0 && c == nchunks - kchunks - 1) FT_EV(tile, 11);
#endif
            tc_fence_after();
            if (elect_one()) {
                if (FT_DEV_BIT(P.debug, 4)) {  // timing experiment: no MMA, hand the slot straight back
                    if constexpr (CG == 1) {
                        mbar_arrive(&empty[stage]);
                    } else {
                        mbar_arrive_cluster(mapa_shared(smem_u32(&empty[stage]), 0));
                        mbar_arrive_cluster(mapa_shared(smem_u32(&empty[stage]), 1));
                    }
                } else {
                    const uint64_t ad = adesc0 + (uint64_t)((stage * C::A_BYTES) >> 4);
                    const uint64_t bd = bdesc0 + (uint64_t)((stage * C::B_BYTES) >> 4);
#pragma unroll
                    for (int kk = 0; kk < BK / UK; ++kk)
                        umma_f16_cg<CG>(d_tmem, ad + (uint64_t)((kk * UK * 2) >> 4),
                                        bd + (uint64_t)((kk * UK * C::WROW) >> 4), C::IDESC, (c | kk) != 0);
                    umma_commit_cg<CG>(&empty[stage]);
                }
            }
            __syncwarp();
            if (++stage == C::STAGES) {
                stage = 0;
                phase ^= 1;
            }
        }
        if ((threadIdx.x & 31) == 0) FT_EV(tile, 7);
        if (elect_one()) {
            if (FT_DEV_BIT(P.debug, 4)) {
                if constexpr (CG == 1) {
                    mbar_arrive(&tfull[acc]);
                } else {
                    mbar_arrive_cluster(mapa_shared(smem_u32(&tfull[acc]), 0));
                    mbar_arrive_cluster(mapa_shared(smem_u32(&tfull[acc]), 1));
                }
            } else {
                umma_commit_cg<CG>(&tfull[acc]);
            }
        }
        __syncwarp();
        acc ^= 1;
        if (acc == 0) acc_phase ^= 1;
    }
    FT_TR_FLUSH((threadIdx.x & 31) == 0);
}

// ------------------------------------------------------------------------------ epilogue
__device__ __forceinline__ uint32_t pack_bf16x2(float lo, float hi) {
    __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);  // RNE
    return *reinterpret_cast<uint32_t*>(&v);
}

// Epilogue warp w reads TMEM lane quadrant w % 4 (rows) and unit range (w - 2) / 4 (U /
// EPI_PARTS of the tile's U units); one thread per batch row.

// Listing 1's linear cell: y = z + s, s = the previous step's output (fp32 ring), 0 at t = 0.
// The 256 accumulator columns are 256 consecutive units; warp half h takes columns h*128 ...
template <int CG, int U>
__device__ __forceinline__ void run_epilogue_linear(const Problem& P, const Tensors& T,
                                                    uint32_t tmem_base, uint64_t* tfull,
                                                    uint64_t* tempty, uint32_t rank) {
    using C = KCfg<CG, U>;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int q = warp & 3, half = (warp - 2) >> 2, row = q * 32 + lane;
    constexpr int COLS = 4 * U / EPI_PARTS;  // accumulator columns per warp
    const bool leader_thread = (threadIdx.x == 64);
    int acc = 0;
    uint32_t acc_phase = 0;
    const int target = flag_target(P);
    __nv_bfloat16* ys = (__nv_bfloat16*)T.h_all;
    TileWalk walk = walk_begin(P, blockIdx.x / CG, gridDim.x / CG);
    TileId tl;
    long long tile;
    while (walk_next(P, walk, tl, tile)) {
        const Cell c = tl.cell;
        int ci = 0, cj = 0;
        const long long cprod = c_producer(P, tl, &ci, &cj);
        const int b = tl.m * ROWS * CG + (int)rank * ROWS + row;
        const bool valid = b < P.B;
        const int n0 = tl.n * 4 * U + half * COLS;
        if (cprod >= 0 && leader_thread)
            wait_flag_geq(T.flags + cprod * P.MB + tl.m, target);
        named_bar_sync(1, EPI_THREADS);
        mbar_wait(&tfull[acc], acc_phase);
        tc_fence_after();
        const uint32_t tbase = tmem_base + (uint32_t)(acc * C::BN) + ((uint32_t)(q * 32) << 16) +
                               (uint32_t)(half * COLS);
        const int row_h = h_row(P, c.d, c.i, c.j, 0);
#pragma unroll 1
        for (int u0 = 0; u0 < COLS; u0 += 16) {
            __syncwarp();
            float z[16];
            tmem_ld_32x32b_x16(tbase + u0, z);
            tmem_wait_ld();
            if (u0 + 16 == COLS) {
                tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if constexpr (CG == 1)
                        mbar_arrive(&tempty[acc]);
                    else
                        mbar_arrive_remote_cta(mapa_shared(smem_u32(&tempty[acc]), 0));
                }
            }
            const int n = n0 + u0;
            if (!valid || n >= P.H) continue;
            if (cprod >= 0) {
#pragma unroll
                for (int v = 0; v < 4; ++v) {
                    const float4 t4 = __ldcg(reinterpret_cast<const float4*>(T.c_ring + c_ring_index(P, c.d, ci, cj, 0, b, n + 4 * v)));
                    z[4 * v] += t4.x;
                    z[4 * v + 1] += t4.y;
                    z[4 * v + 2] += t4.z;
                    z[4 * v + 3] += t4.w;
                }
            }
            uint4 hp[2];
#pragma unroll
            for (int w = 0; w < 2; ++w)
                hp[w] = make_uint4(pack_bf16x2(z[8 * w + 0], z[8 * w + 1]), pack_bf16x2(z[8 * w + 2], z[8 * w + 3]),
                                   pack_bf16x2(z[8 * w + 4], z[8 * w + 5]), pack_bf16x2(z[8 * w + 6], z[8 * w + 7]));
#pragma unroll
            for (int v = 0; v < 4; ++v)
                __stcg(reinterpret_cast<float4*>(T.c_ring + c_ring_index(P, c.d, c.i, c.j, 0, b, n + 4 * v)),
                       make_float4(z[4 * v], z[4 * v + 1], z[4 * v + 2], z[4 * v + 3]));
            uint4* hdst = reinterpret_cast<uint4*>((__nv_bfloat16*)T.hb + hb_row(P, row_h, n / 64, b) * 64 + (n % 64));
            __stcg(hdst, hp[0]);
            __stcg(hdst + 1, hp[1]);
            uint4* ydst = reinterpret_cast<uint4*>(ys + h_all_index(P, c, 0, b, n));
            ydst[0] = hp[0];
            ydst[1] = hp[1];
        }
        named_bar_sync(1, EPI_THREADS);
        if (leader_thread)  // one cumulative release after the barrier: the CTA's EPI_WARPS shares
            red_release_gpu_add(T.flags + cell_lin(P, c.d, c.i, c.j) * P.MB + tl.m, EPI_WARPS);
        acc ^= 1;
        if (acc == 0) acc_phase ^= 1;
    }
}

template <int CG, int U>
__device__ __forceinline__ void run_epilogue(const Problem& P, const Tensors& T, uint32_t tmem_base,
                                             uint64_t* tfull, uint64_t* tempty, uint32_t rank,
                                             float* sbias) {
    using C = KCfg<CG, U>;
    constexpr int EPI_UNITS = C::EPI_UNITS;
    if constexpr (U == 64) {
        if (P.cell == CELL_LINEAR) {
            run_epilogue_linear<CG, U>(P, T, tmem_base, tfull, tempty, rank);
            return;
        }
    }
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int q = warp & 3;                 // TMEM lane quadrant this warp may access
    const int half = (warp - 2) >> 2;       // which unit range of the tile
    constexpr int CH = C::EPI_CH;
    const int row = q * 32 + lane;
    const bool leader_thread = (threadIdx.x == 64);
    int acc = 0;
    uint32_t acc_phase = 0;
    const int target = flag_target(P);
    __nv_bfloat16* h_all = (__nv_bfloat16*)T.h_all;
    __nv_bfloat16* y = (__nv_bfloat16*)T.y;
    __nv_bfloat16* h_n = (__nv_bfloat16*)T.h_n;
    TileWalk walk = walk_begin(P, blockIdx.x / CG, gridDim.x / CG);
    // L2 priority of the nest's live state (the c ring and the blocked h): EVICT_LAST, so the
    // EVICT_FIRST weight stream does not push it out before the next diagonal reads it (ncu, C3:
    // DRAM 30.8 -> 30.1 GB per launch).  FT_DEBUG bit 128 (development builds) reverts to EVICT_NORMAL.
    const uint64_t pol_state = l2_policy((P.l2pol >> 2) & 3,
                                         FT_DEV_BIT(P.debug, 128) ? policy_evict_normal() : policy_evict_last());
    // owner-computes (TileWalk): this thread's rows x units of the slab are the same in every
    // tile, so the cell state stays in registers (cst) from step t to t + 1 — no c ring, no
    // c-ready counter.  Otherwise, under layer bands h and c are published separately ((2b)).
    const int worker = (int)(blockIdx.x / CG), nt0 = nt_layer0(P);
    const bool own = P.owner == 1 || (P.owner == 2 && worker < P.NT) ||
                     (P.owner == 3 && (worker < nt0 || (worker - nt0 < (P.D - 1) * P.NT &&
                                                        P.dil[1 + (worker - nt0) / P.NT] == 1)));
    const bool split = P.band > 0 && !own;
    float cst[EPI_UNITS];
#pragma unroll
    for (int v = 0; v < EPI_UNITS; ++v) cst[v] = 0.f;
    int tcount = 0;
    FT_TR_ROLE;
    TileId tl;
    long long tile;
    while (walk_next(P, walk, tl, tile)) {
        const Cell c = tl.cell;
        int ci = 0, cj = 0;
        const long long cprod = c_producer(P, tl, &ci, &cj);
        const int b = tl.m * ROWS * CG + (int)rank * ROWS + row;
        const bool valid = b < P.B;
        const int n0 = tl.n * U + half * EPI_UNITS;
        FT_TR_DECL;
        // (0) this tile's bias [4 gates][64 units] → shared memory while the MMAs still run (the
        //     L1 is invalidated by every gpu-scope fence, so per-chunk global bias loads would
        //     go to L2 on the epilogue's critical path).  Two buffers, alternating per tile: a
        //     warp can only write tile n+2's buffer after the barrier (1) of tile n+1, which
        //     every warp reaches only after it finished reading tile n's.
        float* sb = sbias + (tcount & 1) * 256;
        ++tcount;
        {
            const int e = threadIdx.x - 64;  // 0 .. 255
            const int slice_b = (P.kind == KIND_SEQ) ? c.d : c.d * 2 + tl.axis;
            // the sigmoid gates' bias is stored halved: σ(z + b) = ½ + ½·tanh(z·½ + b·½), and
            // fma(z, ½, b·½) rounds exactly like ½·(z + b) (power-of-two scaling commutes with RNE)
            if (e < 4 * U)
                sb[e] = __ldg(T.b + ((long long)slice_b * 4 + e / U) * P.H + tl.n * U + e % U) *
                           (e < 3 * U ? 0.5f : 1.0f);
        }
        // (1) the previous cell state, prefetched while this tile's MMAs still run: one acquire
        //     of the c-producer's counter, published to the other epilogue threads by bar.sync
        FT_TR_BEGIN();
        if (cprod >= 0 && leader_thread && !own && !FT_DEV_BIT(P.debug, 1))
            wait_flag_geq(T.flags + (split ? cflag_index(P, cprod, tl.m) : cprod * P.MB + tl.m), target);
        // hb ring (p.hring): this tile's h goes to the slot of step t − len, whose depth consumer
        // (d + 1, t − len) must have read it (its counter completes after its MMAs consumed the
        // operands).  An earlier tile of the wavefront / owner order, so waiting cannot deadlock;
        // it is normally long done (the wait sits before the accumulator wait, off the chain).
        if (P.hring && leader_thread && c.d + 1 < P.D) {
            const int mask = P.hb_mask[c.d];
            if (mask >= 0 && c.i > mask)
                wait_flag_geq(T.flags + cell_lin(P, c.d + 1, c.i - mask - 1, 0) * P.MB + tl.m, target);
        }
        named_bar_sync(1, EPI_THREADS);
        if (leader_thread) FT_TR_END(TR_E_CFLAG);
        // cst: the previous c on entry, updated in place to this tile's c' by the math loop
        // (one register array: the owner walk carries it to the next tile)
        if (own) {
            if (cprod < 0) {
#pragma unroll
                for (int v = 0; v < EPI_UNITS; ++v) cst[v] = 0.f;
            }
        } else if (cprod >= 0 && valid) {
            const float* src = T.c_ring + c_ring_index(P, c.d, ci, cj, tl.axis, b, n0);
            const long long vstride = 4ll * P.B;  // next 4 units of the same batch row
#pragma unroll
            for (int v = 0; v < EPI_UNITS / 4; ++v) {
                const float4 t4 = ld_cg_v4_hint(reinterpret_cast<const float4*>(src + v * vstride), pol_state);
                cst[4 * v + 0] = t4.x;
                cst[4 * v + 1] = t4.y;
                cst[4 * v + 2] = t4.z;
                cst[4 * v + 3] = t4.w;
            }
        } else {
#pragma unroll
            for (int v = 0; v < EPI_UNITS; ++v) cst[v] = 0.f;
        }
        FT_TR_BEGIN();
        mbar_wait(&tfull[acc], acc_phase);
        if (leader_thread) FT_TR_END(TR_E_TFULL);
        if (leader_thread && rank == 0) FT_EV(tile, 3);
        FT_TR_BEGIN();
        tc_fence_after();

        const bool top = (c.d == P.D - 1), last = is_last_pos(P, c);
        const uint32_t tbase = tmem_base + (uint32_t)(acc * C::BN) + ((uint32_t)(q * 32) << 16) +
                               (uint32_t)(half * EPI_UNITS);
        uint4 hp[EPI_UNITS / 8];
        const int row_h = hb_slot_row(P, c.d, c.i, c.j, tl.axis);
#pragma unroll
        for (int u0 = 0; u0 < EPI_UNITS; u0 += CH) {
            __syncwarp();  // tcgen05.ld is .sync.aligned: the whole warp, converged
            float zi[CH], zf[CH], zo[CH], zg[CH];
#ifdef FT_TRACE
            long long _e0 = clock64();
#endif
            tmem_ld_32x32b<CH>(tbase + 0 * U + u0, zi);
            tmem_ld_32x32b<CH>(tbase + 1 * U + u0, zf);
            tmem_ld_32x32b<CH>(tbase + 2 * U + u0, zo);
            tmem_ld_32x32b<CH>(tbase + 3 * U + u0, zg);
            tmem_wait_ld();
            if (u0 == 0 && leader_thread && rank == 0) FT_EV(tile, 13);  // first TMEM chunk in registers
#ifdef FT_TRACE
            if (leader_thread) _acc[TR_E_LDTM] += clock64() - _e0;
            _e0 = clock64();
#endif
            if (u0 + CH == EPI_UNITS) {  // accumulator drained → hand it back to the MMA warp
                tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if constexpr (CG == 1)
                        mbar_arrive(&tempty[acc]);
                    else
                        mbar_arrive_remote_cta(mapa_shared(smem_u32(&tempty[acc]), 0));
                }
            }
            if (FT_DEV_BIT(P.debug, 2)) continue;
            const int ub = half * EPI_UNITS + u0;  // unit offset inside the tile
            float bi[CH], bf[CH], bo[CH], bg[CH];
#pragma unroll
            for (int v = 0; v < CH; v += 4) {
                const float4 t0 = *reinterpret_cast<const float4*>(sb + 0 * U + ub + v);
                const float4 t1 = *reinterpret_cast<const float4*>(sb + 1 * U + ub + v);
                const float4 t2 = *reinterpret_cast<const float4*>(sb + 2 * U + ub + v);
                const float4 t3 = *reinterpret_cast<const float4*>(sb + 3 * U + ub + v);
                bi[v] = t0.x; bi[v + 1] = t0.y; bi[v + 2] = t0.z; bi[v + 3] = t0.w;
                bf[v] = t1.x; bf[v + 1] = t1.y; bf[v + 2] = t1.z; bf[v + 3] = t1.w;
                bo[v] = t2.x; bo[v + 1] = t2.y; bo[v + 2] = t2.z; bo[v + 3] = t2.w;
                bg[v] = t3.x; bg[v + 1] = t3.y; bg[v + 2] = t3.z; bg[v + 3] = t3.w;
            }
            float hv[CH];
#pragma unroll
            for (int v = 0; v < CH; ++v) {
                const float ig = fmaf(0.5f, tanh_approx(fmaf(zi[v], 0.5f, bi[v])), 0.5f);
                const float fg = fmaf(0.5f, tanh_approx(fmaf(zf[v], 0.5f, bf[v])), 0.5f);
                const float og = fmaf(0.5f, tanh_approx(fmaf(zo[v], 0.5f, bo[v])), 0.5f);
                const float gh = tanh_approx(zg[v] + bg[v]);
                const float cn = fmaf(fg, cst[u0 + v], ig * gh);
                cst[u0 + v] = cn;
                hv[v] = og * tanh_approx(cn);
            }
#pragma unroll
            for (int w = 0; w < CH / 8; ++w)
                hp[u0 / 8 + w] = make_uint4(pack_bf16x2(hv[8 * w + 0], hv[8 * w + 1]),
                                            pack_bf16x2(hv[8 * w + 2], hv[8 * w + 3]),
                                            pack_bf16x2(hv[8 * w + 4], hv[8 * w + 5]),
                                            pack_bf16x2(hv[8 * w + 6], hv[8 * w + 7]));
            // what downstream cells read — h (blocked SSA buffer hb) and c (ring) — stored per
            // chunk so the stores overlap the next chunk's math; under layer bands c waits until
            // h is published (see (2b))
            if (valid) {
                const int nn = n0 + u0;
                uint4* hdst = reinterpret_cast<uint4*>(
                    (__nv_bfloat16*)T.hb + hb_row(P, row_h, nn / 64, b) * 64 + (nn % 64));
                if constexpr (CH == 16)
                    st_v8_hint(hdst, hp[u0 / 8], hp[u0 / 8 + 1], pol_state);  // one full sector
                else
                    st_v4_hint(hdst, hp[u0 / 8], pol_state);
                if (!split && !own) {
                    float* cdst = T.c_ring + c_ring_index(P, c.d, c.i, c.j, tl.axis, b, nn);
#pragma unroll
                    for (int v = 0; v < CH / 4; ++v)
                        st_v4_hint(reinterpret_cast<uint4*>(cdst + v * 4ll * P.B),
                                   make_uint4(__float_as_uint(cst[u0 + 4 * v]), __float_as_uint(cst[u0 + 4 * v + 1]),
                                              __float_as_uint(cst[u0 + 4 * v + 2]), __float_as_uint(cst[u0 + 4 * v + 3])),
                                   pol_state);
                }
            }
#ifdef FT_TRACE
            if (leader_thread) _acc[TR_E_MATH] += clock64() - _e0;
#endif
        }
#ifdef FT_TRACE
        long long _e1 = clock64();
#endif
        // (2) publish: each epilogue warp releases its share of the counter as soon as its own
        //     h (and, without bands, c) stores are done — no CTA barrier, so no warp waits for
        //     the slowest one and the release fences of the 8 warps overlap (the counter
        //     completes at CG · EPI_WARPS increments per tile)
        const long long hi = h_all_index(P, c, tl.axis, b, n0);
#ifdef FT_TRACE
        if (leader_thread) _acc[TR_E_STORE] += clock64() - _e1;
        _e1 = clock64();
#endif
        if (leader_thread && rank == 0) FT_EV(tile, 14);  // math and h stores issued (light trace)
        __syncwarp();  // orders the warp's stores before lane 0's release (bar.warp.sync)
#ifdef FT_TRACE
        if (leader_thread) _acc[TR_E_BAR] += clock64() - _e1;
        _e1 = clock64();
#endif
        if (lane == 0) {
            if (P.debug & 64) {  // stress mode (FT_STRESS=1) (tests): a pseudo-random delay before publishing
                const uint32_t h = (uint32_t)(tile * 2654435761u) ^ (uint32_t)(blockIdx.x * 40503u + warp * 977u);
                __nanosleep(200 + (h & 4095u));
            }
            red_release_gpu_add(T.flags + cell_lin(P, c.d, c.i, c.j) * P.MB + tl.m, 1);
        }
        if (leader_thread) {
            FT_TR_END(TR_E_WORK);
            if (rank == 0) FT_EV(tile, 4);
#ifdef FT_TRACE
            _acc[TR_E_REL] += clock64() - _e1;
#endif
        }
        // (2b) layer bands (the h → MMA → epilogue chain is the critical path): the cell state
        //      c' → ring only after h is published, on the c-ready counter (only the
        //      c-consumer's epilogue waits on it, a whole K loop later).  C3 6.61 -> 6.49 ms
        //      same-box; without bands (C4) the extra barrier + release cost more (0.95 -> 0.99)
        if (split && valid) {
            float* cdst = T.c_ring + c_ring_index(P, c.d, c.i, c.j, tl.axis, b, n0);
#pragma unroll
            for (int v = 0; v < EPI_UNITS / 4; ++v)
                st_v4_hint(reinterpret_cast<uint4*>(cdst + v * 4ll * P.B),
                           make_uint4(__float_as_uint(cst[4 * v]), __float_as_uint(cst[4 * v + 1]),
                                      __float_as_uint(cst[4 * v + 2]), __float_as_uint(cst[4 * v + 3])),
                           pol_state);
        }
        if (split) {
            __syncwarp();
            if (lane == 0)
                red_release_gpu_add(T.flags + cflag_index(P, cell_lin(P, c.d, c.i, c.j), tl.m), 1);
        }
        // (3) outputs nobody inside the nest reads
        if (valid) {
            if (h_all) {
                uint4* d = reinterpret_cast<uint4*>(h_all + hi);
#pragma unroll
                for (int w = 0; w < EPI_UNITS / 8; ++w) d[w] = hp[w];
            }
            if (T.c_all) {
                float4* d4 = reinterpret_cast<float4*>(T.c_all + hi);
#pragma unroll
                for (int v = 0; v < EPI_UNITS / 4; ++v)
                    d4[v] = make_float4(cst[4 * v], cst[4 * v + 1], cst[4 * v + 2], cst[4 * v + 3]);
            }
            if (top) {
                uint4* d = reinterpret_cast<uint4*>(y + y_index(P, c, tl.axis, b, n0));
#pragma unroll
                for (int w = 0; w < EPI_UNITS / 8; ++w) d[w] = hp[w];
            }
            if (last) {
                const long long ni = hn_index(P, c, tl.axis, b, n0);
                uint4* d = reinterpret_cast<uint4*>(h_n + ni);
#pragma unroll
                for (int w = 0; w < EPI_UNITS / 8; ++w) d[w] = hp[w];
                float4* d4 = reinterpret_cast<float4*>(T.c_n + ni);
#pragma unroll
                for (int v = 0; v < EPI_UNITS / 4; ++v)
                    d4[v] = make_float4(cst[4 * v], cst[4 * v + 1], cst[4 * v + 2], cst[4 * v + 3]);
            }
        }
        // host-IO overlap: this warp's share of layer d's final state is stored → fence at system
        // scope (a copy engine reads it) and count it for the state copy stream (ft_api.cu hostio)
        if (last && T.nsig) {
            __syncwarp();
            if (lane == 0) {
                fence_acq_rel_sys();
                red_relaxed_sys_add(T.nsig + c.d, 1);
            }
        }
        // (4) host-IO overlap: this warp's share of y(·, t, ·) is stored → fence at system scope
        //     (a copy engine reads it) and count it for the copy stream (ft_api.cu hostio)
        if (top && T.ysig && (P.owner != 1 || c.i % T.ychunk == T.ychunk - 1 || c.i == P.L0 - 1)) {
            // (owner walk: the same warps store every step of their slab, so one fence at the
            //  chunk's last step covers the chunk)
            __syncwarp();
            if (lane == 0) {
                fence_acq_rel_sys();
                red_relaxed_sys_add(T.ysig + c.i / T.ychunk, 1);
            }
        }
        acc ^= 1;
        if (acc == 0) acc_phase ^= 1;
    }
    FT_TR_FLUSH(leader_thread);
}

template <int CG, int U>
__device__ __forceinline__ void kernel_body(const Problem& P, const Tensors& T, const Maps& M) {
    using C = KCfg<CG, U>;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    uint8_t* smem = smem_raw + pad;
    uint8_t* sA = smem;
    uint8_t* sB = smem + C::STAGES * C::A_BYTES;
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES);
    uint64_t* full = bars;
    uint64_t* empty = bars + C::STAGES;
    uint64_t* tfull = bars + 2 * C::STAGES;
    uint64_t* tempty = tfull + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
    float* sbias = reinterpret_cast<float*>(smem + C::STAGES * C::STAGE_BYTES + 256);  // [4][64]

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rank = (CG == 2) ? cluster_ctarank() : 0u;
    FT_TR_ROLE;
    FT_TR_DECL;
    FT_TR_BEGIN();
    if (threadIdx.x == 0) {
        for (int s = 0; s < C::STAGES; ++s) {
            mbar_init(&full[s], 2);  // the leader's weight + activation producers
            mbar_init(&empty[s], 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&tfull[a], 1);
            mbar_init(&tempty[a], EPI_WARPS * CG);
        }
        fence_mbarrier_init();
        tma_prefetch_desc(&M.x);
        tma_prefetch_desc(&M.ys);
        tma_prefetch_desc(&M.h);
        tma_prefetch_desc(&M.W);
        tma_prefetch_desc(&M.U);
    }
    if (warp == 1) tmem_alloc_cg<CG>(tmem_slot, C::TMEM_COLS);
    tc_fence_before();
    __syncthreads();
    if constexpr (CG == 2) cluster_sync();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) run_producer<CG, U, true>(P, T, M, sA, sB, full, empty, rank);
    } else if (warp == 1) {
        if (rank == 0) run_mma<CG, U>(P, tmem_base, sA, sB, full, empty, tfull, tempty);  // whole warp
    } else if (warp == ACT_WARP) {
        if (lane == 0) run_producer<CG, U, false>(P, T, M, sA, sB, full, empty, rank);
    } else {
        run_epilogue<CG, U>(P, T, tmem_base, tfull, tempty, rank, sbias);
    }

    tc_fence_before();
    __syncthreads();
    if constexpr (CG == 2) cluster_sync();
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc_cg<CG>(tmem_base, C::TMEM_COLS);
    }
    if (threadIdx.x == 0) FT_TR_END(TR_TOTAL);
    FT_TR_FLUSH(threadIdx.x == 0);
}

// U0 < U: under owner mode 3 the workers of layer 0 (the only recurrence without slack in a
// dilated nest) run slabs of U0 units — half the MMAs and half the gate math per step on the
// critical chain, and all of a step's recurrent K chunks fit in the deeper ring of the narrower
// stage — with their own tensor maps M0; every other worker runs U-unit slabs.  A CTA's role and
// shared-memory layout are fixed for the whole launch, so each runs one body.
template <int CG, int U, int U0>
__global__ void __launch_bounds__(THREADS, 1)
wavefront_bf16_kernel(const __grid_constant__ Problem P, const __grid_constant__ Tensors T,
                      const __grid_constant__ Maps M, const __grid_constant__ Maps M0) {
    if constexpr (U0 != U) {
        if (P.owner == 3 && (int)(blockIdx.x / CG) < P.nt0) {
            kernel_body<CG, U0>(P, T, M0);
            return;
        }
    }
    kernel_body<CG, U>(P, T, M);
}

// ------------------------------------------------------------------------------ host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode_fn(std::string* err) {
    static EncodeTiledFn fn = nullptr;
    if (fn) return fn;
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q = cudaDriverEntryPointSymbolNotFound;
    cudaError_t e = cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &ptr, 12000,
                                                     cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !ptr) {
        if (err) *err = "cuTensorMapEncodeTiled not available from the driver";
        return nullptr;
    }
    fn = reinterpret_cast<EncodeTiledFn>(ptr);
    return fn;
}

// Blocked activation view (64 units, rows) with a (64, 128) box: one box = one contiguous 16 KiB
// K-chunk of 128 batch rows.
bool encode_blocked(EncodeTiledFn enc, CUtensorMap* m, const void* base, long long rows,
                    std::string* err) {
    const cuuint64_t dims[2] = {64, (cuuint64_t)rows};
    const cuuint64_t strides[1] = {128};
    const cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)ROWS};
    const cuuint32_t es[2] = {1, 1};
    CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides,
                     box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
        if (err) *err = "cuTensorMapEncodeTiled(blocked activation) failed: " + std::to_string((int)r);
        return false;
    }
    return true;
}

// Weight view (n, k, gate, slice) with a (64, 64, gates, 1) box, 128-byte swizzle: the box is
// the [i | f | o | ĝ] (CG 1) or [i | f] / [o | ĝ] (CG 2) x 64-unit slab of one 64-row K chunk.
bool encode_wt(EncodeTiledFn enc, CUtensorMap* m, const void* base, int H, int krows, int slices,
               int gates, int units, std::string* err) {
    const cuuint64_t dims[4] = {(cuuint64_t)H, (cuuint64_t)krows, 4, (cuuint64_t)slices};
    const cuuint64_t strides[3] = {(cuuint64_t)H * 2, (cuuint64_t)krows * H * 2,
                                   (cuuint64_t)4 * krows * H * 2};
    const cuuint32_t box[4] = {(cuuint32_t)units, (cuuint32_t)BK, (cuuint32_t)gates, 1};
    const cuuint32_t es[4] = {1, 1, 1, 1};
    CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(base), dims, strides,
                     box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     units == 64 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
        if (err) *err = "cuTensorMapEncodeTiled(weight) failed: " + std::to_string((int)r);
        return false;
    }
    return true;
}

// The device's persisting-L2 set-aside (cudaLimitPersistingL2CacheSize) is raised once to what
// the window needs and then left alone (it is device-wide; lowering it would evict other users'
// persisting lines).  Never changed while `s` is being captured into a graph.
bool persisting_limit_at_least(int dev, size_t bytes, cudaStream_t s) {
    static size_t set_to[64] = {0};
    if (dev < 0 || dev >= 64) return false;
    if (set_to[dev] >= bytes) return true;
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(s, &cs) != cudaSuccess || cs != cudaStreamCaptureStatusNone) {
        cudaGetLastError();
        return false;
    }
    size_t cur = 0;
    if (cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize) == cudaSuccess && cur >= bytes) {
        set_to[dev] = cur;
        return true;
    }
    if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, bytes) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    set_to[dev] = bytes;
    return true;
}

// Layer bands (a5 when the weight set does not fit in L2, e.g. C3's 256 MiB): the stacked nest
// runs band after band of `band` layers (ft_common.cuh next_cell), so one diagonal reads only the
// band's weights — 4 x 16 MiB at H = 1024 — and those stay in L2 (EVICT_LAST) for the band's
// T + band - 1 diagonals instead of streaming from HBM on every diagonal.  The price is a longer
// dependency chain (D / band · (T + band − 1) diagonals instead of T + D − 1) and fewer cells per
// diagonal; the band is the largest whose weights fit in a 64 MiB L2 budget (measured: 5-6 layers
// of 16 MiB no longer stay resident) and it is used only when a band's diagonal still gives at
// least 3/4 of the CTA groups a tile.  C3 (same box): 7.44 -> 6.57 ms, the SM clock at the power
// cap 997 -> 1455 MHz (profiles/r2_band_sweep.txt).  FT_BAND overrides (0 = off).
int choose_band(const Problem& p, int workers) {
    if (p.cell != CELL_LSTM) return 0;
    if (const char* e = getenv("FT_BAND")) {
        const int b = atoi(e);
        return b > 0 && b < p.D ? b : 0;
    }
    if (p.kind == KIND_GRID) {
        // grid nests carry two fp32 cell states per cell (c^x, c^y): one slot per column / row
        // and depth, (Lx + Ly) slots of B·H fp32 per depth.  A depth band's live L2 set is its
        // rings, its weights (2 axes x 4 gates x H x 3H bf16 per depth) and the SSA rows it
        // streams; when the whole nest's set exceeds the budget, run depth bands whose rings and
        // weights fit in 40 MiB.  C5: 16 + 12 MiB per depth -> bands of 1.  Same box: DRAM 9.6 GB
        // (paper order, 2-slot rings) -> 5.9 GB (bands of 2) -> 2.95 GB (bands of 1) -> 2.33 GB
        // (bands of 1, 1-slot rings) per forward, time unchanged; bands of 2 with 1-slot rings
        // spill again (4.5 GB) at the same time (profiles/r2_ab_grid_bands.txt,
        // profiles/rnd2_ab_c5_band1.txt, profiles/rnd2_ab_c5_cring.txt)
        const double ring_per_depth = (double)(p.L0 + p.L1) * (double)p.B * p.H * 4.0;
        const double w_per_depth = 2.0 * 4.0 * p.H * 3.0 * p.H * 2.0;
        const double per_depth = ring_per_depth + w_per_depth;
        const double budget = 40.0 * 1024 * 1024;
        if (per_depth * p.D <= budget) return 0;
        const int band = (int)(budget / per_depth);
        return band < 1 ? 1 : (band >= p.D ? 0 : band);
    }
    if (p.kind != KIND_SEQ) return 0;
    if (p.resident_layers >= p.D) return 0;  // the whole weight set already stays in L2
    const double layer_bytes = 8.0 * p.H * p.H * 2.0;  // W + U of one layer, bf16
    const int band = (int)((64.0 * 1024 * 1024) / layer_bytes);
    if (band < 1 || band >= p.D) return 0;
    if (4ll * band * p.NT * p.MB < 3ll * workers) return 0;
    return band;
}

// Host-side launch state cached across calls (serving loops call the same shapes with the same
// buffers over and over): the tensor maps per (buffers, shape), and per device the dynamic
// shared-memory attribute and the cluster occupancy.  Keys hold every input of the encoding, so
// a hit returns exactly what a fresh encode would.
struct MapsKey {
    const void *x, *ys, *W, *U, *hb, *xb, *yb;
    int kind, cell, B, L0, L1, H, D, MB, BM, x_direct, cg, units, dev;
    bool operator==(const MapsKey& o) const { return std::memcmp(this, &o, sizeof(MapsKey)) == 0; }
};
struct MapsCache {
    static constexpr int N = 8;
    std::mutex mu;
    MapsKey key[N];
    Maps maps[N];
    int used = 0, next = 0;
    bool find(const MapsKey& k, Maps* out) {
        std::lock_guard<std::mutex> g(mu);
        for (int i = 0; i < used; ++i)
            if (key[i] == k) {
                *out = maps[i];
                return true;
            }
        return false;
    }
    void put(const MapsKey& k, const Maps& m) {
        std::lock_guard<std::mutex> g(mu);
        key[next] = k;
        maps[next] = m;
        next = (next + 1) % N;
        if (used < N) ++used;
    }
};
MapsCache& maps_cache() {
    static MapsCache c;
    return c;
}

template <int CG, int U>
cudaError_t encode_maps(const Problem& p, const Tensors& t, EncodeTiledFn enc, bool x_direct, Maps* Mp,
                        std::string* err) {
    using C = KCfg<CG, U>;
    Maps& M = *Mp;
    const int slices = p.D * p.naxes;
    const int Bp = p.MB * p.BM;
    if (!encode_blocked(enc, &M.x, t.xb, (long long)p.L0 * (p.H / 64) * Bp, err)) return cudaErrorInvalidValue;
    // Stacked/dilated: layer-0 inputs are read straight from x [B][T][H] (3-D TMA, 128 rows of
    // 128 B per box) instead of being packed into the blocked layout first: the pack launch goes
    // away and the strided loads are off the dependency chain (x has no producer).  Same-box
    // C3 5.44 -> 5.40 ms, C4 0.922 -> 0.903 ms (profiles/r2_ab_x_direct.txt).  Grid inputs are
    // still packed.  FT_X_DIRECT=0 restores the pack (A/B).
    M.xd = M.x;
    if (x_direct) {
        const cuuint64_t dims[3] = {(cuuint64_t)p.H, (cuuint64_t)p.L0, (cuuint64_t)p.B};
        const cuuint64_t strides[2] = {(cuuint64_t)p.H * 2, (cuuint64_t)p.L0 * p.H * 2};
        const cuuint32_t box[3] = {(cuuint32_t)BK, 1, (cuuint32_t)ROWS};
        const cuuint32_t es[3] = {1, 1, 1};
        CUresult r = enc(&M.xd, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(t.x), dims, strides,
                         box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                         CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) {
            if (err) *err = "cuTensorMapEncodeTiled(direct x) failed: " + std::to_string((int)r);
            return cudaErrorInvalidValue;
        }
    }
    if (!encode_blocked(enc, &M.ys, p.kind == KIND_GRID ? t.yb : t.xb,
                        (long long)(p.kind == KIND_GRID ? p.L1 : p.L0) * (p.H / 64) * Bp, err))
        return cudaErrorInvalidValue;
    if (!encode_blocked(enc, &M.h, t.hb, hb_rows_total(p), err)) return cudaErrorInvalidValue;
    if (p.cell == CELL_LINEAR) {
        // W [D][H][H] as (64 n_lo, k, H/64 n_hi, d): a box of 4 (or 2) 64-unit atoms is the
        // 256-unit N tile of one 64-deep K chunk — the same SMEM layout as the LSTM gate atoms
        const cuuint64_t dims[4] = {64, (cuuint64_t)p.H, (cuuint64_t)(p.H / 64), (cuuint64_t)p.D};
        const cuuint64_t strides[3] = {(cuuint64_t)p.H * 2, 128, (cuuint64_t)p.H * p.H * 2};
        const cuuint32_t box[4] = {64, (cuuint32_t)BK, (cuuint32_t)C::GATES, 1};
        const cuuint32_t es[4] = {1, 1, 1, 1};
        CUresult r = enc(&M.W, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(t.W), dims, strides,
                         box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                         CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) {
            if (err) *err = "cuTensorMapEncodeTiled(linear weight) failed: " + std::to_string((int)r);
            return cudaErrorInvalidValue;
        }
        M.U = M.W;
    } else {
        if (!encode_wt(enc, &M.W, t.W, p.H, p.H, slices, C::GATES, U, err)) return cudaErrorInvalidValue;
        if (!encode_wt(enc, &M.U, t.U, p.H, u_krows(p), slices, C::GATES, U, err))
            return cudaErrorInvalidValue;
    }

    return cudaSuccess;
}

template <int CG, int U>
cudaError_t launch_cg_maps(const Problem& p, const Tensors& t, cudaStream_t s, std::string* err,
                           const Maps& M, const Maps* M0, bool x_direct, int dev, int nsm, int* clusters) {
    using C = KCfg<CG, U>;
    cudaError_t e = cudaSuccess;
    const int Bp = p.MB * p.BM;
    // layer-0 inputs → blocked layout (part of the forward; ~T*H*Bp*4 bytes of traffic)
    {
        const long long nvec = (long long)p.L0 * (p.H / 64) * Bp * 8;
        const int blocks = (int)((nvec + 255) / 256 < 4 * nsm ? (nvec + 255) / 256 : 4 * nsm);
        if (!x_direct)
            pack_rows_kernel<<<blocks, 256, 0, s>>>((const __nv_bfloat16*)t.x, (__nv_bfloat16*)t.xb, p.B, p.L0, p.H, Bp);
        if (p.kind == KIND_GRID) {
            const long long nv2 = (long long)p.L1 * (p.H / 64) * Bp * 8;
            const int b2 = (int)((nv2 + 255) / 256 < 4 * nsm ? (nv2 + 255) / 256 : 4 * nsm);
            pack_rows_kernel<<<b2, 256, 0, s>>>((const __nv_bfloat16*)t.ys, (__nv_bfloat16*)t.yb, p.B, p.L1, p.H, Bp);
        }
        e = cudaGetLastError();
        if (e != cudaSuccess) {
            if (err) *err = std::string("input pack launch: ") + cudaGetErrorString(e);
            return e;
        }
    }
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(THREADS);
    cfg.dynamicSmemBytes = C::SMEM_BYTES;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    long long grid;
    if constexpr (CG == 1) {
        grid = nsm;
        if (grid > p.ntiles) grid = p.ntiles;
        attr[0].id = cudaLaunchAttributeCooperative;  // all CTAs co-resident (spin-wait safety)
        attr[0].val.cooperative = 1;
    } else {
        // Cluster launch: every cluster must be co-resident; size the grid by the number of
        // clusters the device can hold at once (one CTA per SM, so <= nsm / 2).
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = 2;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        cfg.gridDim = dim3((unsigned)(nsm & ~1));
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        int nclusters = clusters[dev];
        if (nclusters < 1) {
            e = cudaOccupancyMaxActiveClusters(&nclusters, wavefront_bf16_kernel<CG, U, U>, &cfg);
            if (e != cudaSuccess || nclusters < 1) {
                if (err) *err = std::string("cluster occupancy query: ") + cudaGetErrorString(e);
                return e != cudaSuccess ? e : cudaErrorInvalidConfiguration;
            }
            clusters[dev] = nclusters;
        }
        grid = 2ll * nclusters;
        if (grid > 2 * p.ntiles) grid = 2 * p.ntiles;
    }
    cfg.gridDim = dim3((unsigned)grid);
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    // Persisting L2 window over W of the first layers (streaming regime only: the weight set does
    // not fit in L2, so every diagonal re-reads it from DRAM).  The window's layers are read from
    // L2 on every diagonal after the first; their TMA loads carry EVICT_NORMAL so the hint does
    // not fight the window.  C3: DRAM 31.5 -> 28.5 GB per forward, -3 % time at the power cap
    // (profiles/r2_ab_l2_persist.jsonl).  ft_set_l2_persist() sizes or disables it.
    Problem q = p;
    q.persist_layers = 0;
    q.flag_mult = CG * EPI_WARPS;  // every epilogue warp of every CTA of a tile releases once
    q.x_direct = x_direct;
    q.band = choose_band(p, (int)(grid / CG));
    if (q.hring) hb_layout(q, q.band);
    // Dedicated owners for layer 0 of a dilated nest (TileWalk owner mode 2): layer 0 has
    // dilation 1, the only recurrence without slack, so its slabs get their own CTA pairs (cell
    // state in registers, no queueing behind other layers' tiles); the other layers run
    // round-robin on the rest.  Round 1 measured it slower (C4 0.916 -> 0.958 ms); with the
    // round-2 epilogue and launch path it is faster: C4 0.838 -> 0.798 ms same-box
    // (profiles/rnd2_ab_c4_owner_l0.txt).  Default for dilated nests; FT_OWNER_L0=0 turns it off.
    {
        bool dilated = false;
        for (int d = 1; d < p.D; ++d) dilated = dilated || p.dil[d] > 1;
        const char* e = getenv("FT_OWNER_L0");
        const bool want = e ? atoi(e) != 0 : dilated;
        if (want && q.band == 0 && p.kind == KIND_SEQ && p.cell == CELL_LSTM && p.MB == 1 &&
            p.naxes == 1 && p.D >= 2 && p.dil[0] == 1 && 2ll * p.NT <= grid / CG)
            q.owner = 2;
        // every layer owned (TileWalk mode 3) when all D·NT slabs get a pair: each layer then
        // advances at the pace of the layer below with a constant lag instead of queueing behind
        // other layers' tiles (C4 0.750 -> 0.737 ms pipelined same-box,
        // profiles/rnd2_ab_owner_all.txt); FT_OWNER_ALL=0 keeps mode 2
        const char* ea = getenv("FT_OWNER_ALL");
        if (q.owner == 2 && !(ea && ea[0] == '0') && (long long)p.D * p.NT <= grid / CG) q.owner = 3;
        // ... and layer 0 in half-width slabs (wavefront_bf16_kernel<2, 64, 32>) when those fit
        // too; FT_NARROW0=0 keeps layer 0 at the common width
        if constexpr (CG == 2 && U == 64) {
            const char* en = getenv("FT_NARROW0");
            const int nt0 = p.H / 32;
            if (q.owner == 3 && M0 && !(en && en[0] == '0') && nt0 + (long long)(p.D - 1) * p.NT <= grid / CG)
                q.nt0 = nt0;
        }
    }
    // recurrent half first for dilated layers (segments); FT_REC_FIRST=0 keeps the input half first
    {
        const char* e = getenv("FT_REC_FIRST");
        q.rec_first = !(e && e[0] == '0');
    }
#ifdef FT_DEV_EXPERIMENTS
    if (const char* e = getenv("FT_L2POL")) q.l2pol = atoi(e);  // L2 policy experiments (dev builds)
#endif
    if (q.band > 0) {
        q.resident_layers = p.D;  // every band's weights EVICT_LAST: resident while the band runs
        bool unit_dil = true;
        for (int d = 0; d < p.D; ++d) unit_dil = unit_dil && p.dil[d] == 1;
        q.owner = unit_dil && p.MB == 1 && p.naxes == 1 && (long long)q.band * p.NT <= grid / CG;
        if (const char* e = getenv("FT_OWNER")) q.owner = q.owner && atoi(e) != 0;  // A/B
        if (const char* e = getenv("FT_SKEW")) q.skew = atoi(e);
    }
    cudaLaunchAttribute attr2[2];
    int nattr = 1;
    if (q.band == 0 && p.resident_layers == 0 && p.kind == KIND_SEQ && p.cell == CELL_LSTM &&
        p.persist_layers != 0) {
        int maxp = 0, maxw = 0;
        cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev);
        cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, dev);
        const size_t layer_bytes = (size_t)4 * p.H * p.H * 2;
        const long long mib = l2_persist_mib();
        size_t budget = mib >= 0 ? (size_t)mib << 20 : (size_t)48 << 20;  // auto: 48 MiB (measured)
        if (budget > (size_t)maxp * 6 / 10) budget = (size_t)maxp * 6 / 10;
        if (budget > (size_t)maxw) budget = (size_t)maxw;
        int k = (int)(budget / layer_bytes);
        if (p.persist_layers > 0) k = p.persist_layers;  // FT_L2_PERSIST_LAYERS (experiments)
        if (k > p.D) k = p.D;
        size_t bytes = (size_t)k * layer_bytes;
        if (bytes > (size_t)maxw) { k = (int)((size_t)maxw / layer_bytes); bytes = (size_t)k * layer_bytes; }
        if (k > 0 && maxp > 0 && persisting_limit_at_least(dev, bytes < (size_t)maxp ? bytes : (size_t)maxp, s)) {
            const size_t lim = bytes < (size_t)maxp ? bytes : (size_t)maxp;
            q.persist_layers = k;
            attr2[0] = attr[0];
            attr2[1].id = cudaLaunchAttributeAccessPolicyWindow;
            attr2[1].val.accessPolicyWindow.base_ptr = const_cast<void*>(t.W);
            attr2[1].val.accessPolicyWindow.num_bytes = bytes;
            attr2[1].val.accessPolicyWindow.hitRatio = (float)lim / (float)bytes;
            attr2[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
            attr2[1].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
            cfg.attrs = attr2;
            cfg.numAttrs = 2;
            nattr = 2;
        }
    }
    if (t.ysig_per_step) {  // every epilogue warp of every tile of a top-layer cell signals once
        *t.ysig_per_step = (t.ysig && q.kind == KIND_SEQ && q.cell == CELL_LSTM)
                               ? q.naxes * q.MB * q.NT * CG * EPI_WARPS : 0;
        if (t.ysig_per_chunk) *t.ysig_per_chunk = q.owner == 1;  // owner walk: once per chunk
        if (t.nsig0_per_step)  // layer 0's final-state count when it runs narrower slabs
            *t.nsig0_per_step = (*t.ysig_per_step && q.nt0 > 0) ? q.naxes * q.MB * q.nt0 * CG * EPI_WARPS : 0;
    }
    auto kern = wavefront_bf16_kernel<CG, U, U>;
    const Maps* m0 = &M;
    if constexpr (CG == 2 && U == 64) {
        if (q.nt0 > 0) {
            kern = wavefront_bf16_kernel<2, 64, 32>;
            m0 = M0;
            static bool set_mixed[64] = {};
            if (!set_mixed[dev]) {
                e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM_BYTES);
                if (e != cudaSuccess) {
                    if (err) *err = std::string("bf16 launch setup (narrow layer 0): ") + cudaGetErrorString(e);
                    return e;
                }
                set_mixed[dev] = true;
            }
        }
    }
    int coop = 1;
    if constexpr (CG == 2)
        e = launch_cluster_persistent(cfg, nattr == 2 ? attr2 : attr, nattr, &coop, kern, q, t, M, *m0);
    else
        e = cudaLaunchKernelEx(&cfg, kern, q, t, M, *m0);
    if (e == cudaSuccess)
        set_last_launch("wavefront_bf16_kernel<" + std::to_string(CG) + "," + std::to_string(U) +
                        (q.nt0 > 0 ? ",32" : "") +
                        "> grid=" + std::to_string(grid) + " cluster=" + std::to_string(CG) +
                        " cooperative=" + std::to_string(coop) + " band=" + std::to_string(q.band) +
                        " skew=" + std::to_string(seq_skew(q)) + " owner=" + std::to_string(q.owner) +
                        " nt0=" + std::to_string(nt_layer0(q)) +
                        " x_direct=" + std::to_string(q.x_direct) + " persist_layers=" +
                        std::to_string(q.persist_layers) + " resident_layers=" +
                        std::to_string(q.resident_layers) + " stress=" + std::to_string((q.debug & 64) != 0));
    if (e != cudaSuccess && err) *err = std::string("bf16 launch: ") + cudaGetErrorString(e);
    return e;
}

template <int CG, int U>
cudaError_t launch_cg(const Problem& p, const Tensors& t, cudaStream_t s, std::string* err) {
    using C = KCfg<CG, U>;
    EncodeTiledFn enc = get_encode_fn(err);
    if (!enc) return cudaErrorNotSupported;
    int dev = 0, nsm = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess || dev < 0 || dev >= 64) {
        if (err) *err = std::string("bf16 launch setup: ") + cudaGetErrorString(e);
        return e != cudaSuccess ? e : cudaErrorInvalidDevice;
    }
    const char* exd = getenv("FT_X_DIRECT");
    const bool x_direct = p.kind == KIND_SEQ && (t.xsig != nullptr || !(exd && exd[0] == '0'));
    MapsKey key;
    std::memset(&key, 0, sizeof(key));
    key = MapsKey{t.x, t.ys, t.W, t.U, t.hb, t.xb, t.yb, p.kind, p.cell, p.B, p.L0, p.L1, p.H, p.D,
                  p.MB, p.BM, (int)x_direct, CG, U, dev};
    Maps M;
    if (!maps_cache().find(key, &M)) {
        const cudaError_t ee = encode_maps<CG, U>(p, t, enc, x_direct, &M, err);
        if (ee != cudaSuccess) return ee;
        maps_cache().put(key, M);
    }
    // per-device one-time setup: the shared-memory opt-in and the cluster occupancy
    static bool attr_set[64] = {};
    static int clusters[64] = {};
    if (!attr_set[dev]) {
        e = cudaFuncSetAttribute(wavefront_bf16_kernel<CG, U, U>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 C::SMEM_BYTES);
        if (e != cudaSuccess) {
            if (err) *err = std::string("bf16 launch setup: ") + cudaGetErrorString(e);
            return e;
        }
        attr_set[dev] = true;
    }
    // narrow layer-0 slabs (owner mode 3 of a dilated nest): tensor maps of the 32-unit tile
    Maps M0;
    const Maps* m0 = nullptr;
    if constexpr (CG == 2 && U == 64) {
        bool dilated = false;
        for (int d = 1; d < p.D; ++d) dilated = dilated || p.dil[d] > 1;
        if (dilated && p.kind == KIND_SEQ && p.cell == CELL_LSTM && p.dil[0] == 1 && p.H % 64 == 0) {
            MapsKey k0 = key;
            k0.units = 32;
            if (!maps_cache().find(k0, &M0)) {
                const cudaError_t ee = encode_maps<2, 32>(p, t, enc, x_direct, &M0, err);
                if (ee != cudaSuccess) return ee;
                maps_cache().put(k0, M0);
            }
            m0 = &M0;
        }
    }
    return launch_cg_maps<CG, U>(p, t, s, err, M, m0, x_direct, dev, nsm, clusters);
}

}  // namespace

#ifdef FT_TRACE
extern "C" __attribute__((visibility("default"))) int ft_debug_trace(unsigned long long* host,
                                                                     int n, int reset) {
    if (n > 1024 * TR_SLOTS) n = 1024 * TR_SLOTS;
    cudaDeviceSynchronize();
    if (cudaMemcpyFromSymbol(host, g_trace, n * sizeof(unsigned long long)) != cudaSuccess) return -1;
    if (reset) {
        static unsigned long long zeros[1024 * TR_SLOTS];
        cudaMemcpyToSymbol(g_trace, zeros, sizeof(zeros));
    }
    return TR_SLOTS;
}
#endif
#if defined(FT_TRACE) || defined(FT_TRACE_LIGHT)
extern "C" __attribute__((visibility("default"))) int ft_debug_events(unsigned long long* host, int ntiles) {
    if (ntiles > EV_MAX_TILES) ntiles = EV_MAX_TILES;
    cudaDeviceSynchronize();
    if (cudaMemcpyFromSymbol(host, g_events, (size_t)ntiles * EV_K * sizeof(unsigned long long)) != cudaSuccess) return -1;
    return ntiles;
}
#endif

bool hb_ring_eligible(const Problem& p) {
    if (p.kind != KIND_SEQ || p.cell != CELL_LSTM) return false;
    if (p.B <= ROWS && resident_bnu(p, 148) != 0) return false;  // SMEM-resident candidate
    if (p.B <= 64 && (p.H == 128 || p.H == 256)) return false;    // DSMEM-cluster candidate
    return true;
}

int bf16_kernel_choice(const Problem& p) {
    if (p.hring) return 2;  // laid out for the streaming kernel (hb_ring_eligible)
    // latency-bound small stacked LSTMs (C2): weights resident in the SMEM of one cluster per
    // layer, h exchanged through DSMEM on the time edge (wavefront_cluster.cu)
    const char* envc = getenv("FT_CLUSTER");  // "0" disables it (comparisons)
    const char* env = getenv("FT_RESIDENT");  // "0" forces the streaming kernel (comparisons)
    if (!(envc && envc[0] == '0') && !(env && env[0] == '0') && cluster_kernel_applies(p)) return 0;
    // a5: weights resident in shared memory for the whole sequence when they fit
    if (p.BM == ROWS && !(env && env[0] == '0')) {
        int dev = 0, nsm = 0;
        if (cudaGetDevice(&dev) == cudaSuccess &&
            cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess &&
            resident_bnu(p, nsm))
            return 1;
    }
    return 2;
}

cudaError_t launch_wavefront_bf16(const Problem& p, const Tensors& t, cudaStream_t s,
                                  std::string* err) {
    const int choice = bf16_kernel_choice(p);
    if (choice == 0) return launch_wavefront_cluster(p, t, s, err);
    if (choice == 1) {
        int dev = 0, nsm = 148;
        if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        return launch_wavefront_resident(p, t, s, resident_bnu(p, nsm), err);
    }
    // N-tile width: 64 units by default; 32 units only when a diagonal at 64 units would give
    // under a quarter of the CTA groups a tile: twice the tiles, half the per-tile latency on the
    // dependency chain, but 1.5x the operand traffic per FLOP.
    const int cg = p.BM == 2 * ROWS ? 2 : 1;
    int dev = 0, nsm = 148;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    long long max_cells = 0;
    if (p.kind == KIND_SEQ) {
        max_cells = p.D < p.L0 ? p.D : p.L0;
    } else {
        for (int k = 0; k < p.D + p.L0 + p.L1 - 2; ++k) {
            long long n = 0;
            for (int d = 0; d < p.D && d <= k; ++d) {
                const int r = k - d;
                const int ilo = r - (p.L1 - 1) > 0 ? r - (p.L1 - 1) : 0, ihi = r < p.L0 - 1 ? r : p.L0 - 1;
                if (ihi >= ilo) n += ihi - ilo + 1;
            }
            if (n > max_cells) max_cells = n;
        }
    }
    // (round 2: with the leaner epilogue and tile decode, 64-unit tiles beat 32-unit ones on C4
    //  — 0.902 -> 0.852 ms — although its diagonals give only 48 of 74 CTA pairs a tile; the
    //  32-unit split now only pays on diagonals a quarter of that wide)
    int units = (4 * max_cells * p.naxes * p.MB * p.NT < nsm / cg && p.cell == CELL_LSTM && p.H % 32 == 0) ? 32 : 64;
    if (const char* env = getenv("FT_TILE_UNITS")) units = atoi(env) == 32 && p.cell == CELL_LSTM ? 32 : 64;
    if (units == 64)
        return cg == 2 ? launch_cg<2, 64>(p, t, s, err) : launch_cg<1, 64>(p, t, s, err);
    Problem q = p;
    q.BNU = 32;
    q.NT = p.H / 32;
    q.ntiles = q.ncells * q.naxes * q.MB * q.NT;
    return cg == 2 ? launch_cg<2, 32>(q, t, s, err) : launch_cg<1, 32>(q, t, s, err);
}

}  // namespace ft
