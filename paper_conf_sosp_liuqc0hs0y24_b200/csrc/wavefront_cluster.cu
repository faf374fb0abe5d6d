// wavefront_cluster.cu — the latency-bound stacked LSTM (e.g. C2) with the recurrent state
// exchanged through distributed shared memory.
//
// In a wavefront every monotone path from cell (0, 0) to (D-1, T-1) has exactly T-1 time edges
// (h_{d,t-1} → cell (d, t), Listing 2) and D-1 depth edges (h_{d-1,t} → cell (d, t),
// Listing 1), so the critical path is (T-1)·latency(time edge) + (D-1)·latency(depth
// edge) (Table 4 dependence vectors, L307–L317).  With T ≫ D the time edge dominates.  Here one
// layer's hidden units are split over a thread-block cluster (H/32 CTAs, 32 units each) whose
// CTAs keep their weight slab resident in shared memory (the reuse of L345–L349, as in
// wavefront_resident.cu) and hand h_{d,t} to each other through DSMEM: every epilogue thread
// writes its row of the CTA's 32-unit slice of h_{d,t} straight from registers into every cluster
// CTA's recurrent operand buffer (st.async shared::cluster, each store carrying complete_tx to the
// receiver's mbarrier).  The receiver's MMA warp waits on that mbarrier — no global-memory round
// trip, no readiness counter, no staging or CTA barrier on the time edge.  (A first version
// staged the slice and bulk-copied it, cp.async.bulk shared::cluster: 0.77 us more per step.)  Depth edges (layer d-1 → d, another cluster) still go through the blocked
// SSA buffer hb + a release/acquire counter, as in the other kernels.
//
// Shapes: batch B <= 64 (the tile is M = 128 with rows >= B never stored), H in {128, 256}
// (cluster of H/32 <= 8 CTAs), stacked (dilation 1).  N = 4 gates x 32 units = 128, K = 64 per
// chunk.  Warps: 0 TMA producer, 1 MMA issuer (whole warp), 4, 5, 8, 9 epilogue (the warps of
// TMEM lane quadrants 0 and 1, i.e. rows 0..63, two per quadrant with 16 units each).
//
// Recurrent operand layout (no swizzle, K-major): k-group g (8 units, 16 bytes) of all 64 rows is
// one contiguous 1 KiB block (row r at r*16), so CTA j's 32 units = k-groups 4j..4j+3 = ONE
// contiguous 4 KiB run in every receiver.  UMMA descriptor: core matrix = 8 rows x 16 B
// (128 contiguous bytes), LBO = 1 KiB (next core matrix along K), SBO = 128 B (next 8 rows).
// Rows 64..127 of the M = 128 operand read the next k-group's block (or the following buffer):
// garbage rows whose accumulator lanes are never read.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <string>

#include "ft_internal.h"
#include "ft_sm100.cuh"

namespace ft {

#ifdef FT_TRACE
// development-only (libft_trace.so): per-step %globaltimer stamps of CTA `g_cev_cta`:
// 0 MMA warp saw hfull, 1 MMA warp committed, 2 epilogue saw tfull, 3 math done, 4 copies issued,
// 5 x-half ready (MMA warp saw the first xfull of the step); 4 = the sends were issued
__device__ unsigned long long g_cev[4096 * 8];
__device__ int g_cev_cta = 0;
#define FT_CEV(t, k) do { if (blockIdx.x == g_cev_cta && (t) < 4096) g_cev[(t) * 8 + (k)] = globaltimer_ns(); } while (0)
// per layer: %globaltimer when slice 0's epilogue saw the accumulator of step t (all layers, one run)
__device__ unsigned long long g_lev[64 * 1024];
#define FT_LEV(d, t) do { if ((d) < 64 && (t) < 1024) g_lev[(d) * 1024 + (t)] = globaltimer_ns(); } while (0)
extern "C" __attribute__((visibility("default"))) int ft_debug_cluster_layer_events(unsigned long long* host, int D, int T) {
    cudaDeviceSynchronize();
    for (int d = 0; d < D && d < 64; ++d)
        if (cudaMemcpyFromSymbol(host + (size_t)d * T, g_lev, (size_t)T * 8, (size_t)d * 1024 * 8) != cudaSuccess) return -1;
    return D;
}
extern "C" __attribute__((visibility("default"))) int ft_debug_cluster_events(unsigned long long* host, int nsteps, int cta) {
    if (nsteps > 4096) nsteps = 4096;
    cudaDeviceSynchronize();
    if (cudaMemcpyFromSymbol(host, g_cev, (size_t)nsteps * 8 * 8) != cudaSuccess) return -1;
    cudaMemcpyToSymbol(g_cev_cta, &cta, sizeof(int));
    return nsteps;
}
#else
#define FT_CEV(t, k) ((void)0)
#define FT_LEV(d, t) ((void)0)
#endif

namespace {

using namespace sm100;

constexpr int KROWS = 128;  // UMMA M
constexpr int KB = 64;      // batch rows actually carried (B <= KB)
constexpr int KBK = 64;     // K per chunk
// 10 warps: 0 TMA, 1 MMA, and the epilogue warps whose TMEM lane quadrant (warp % 4) holds the
// batch rows 0..63 — warps 4, 5 (the first half of the CTA's units) and 8, 9 (the second half).
// Warps 2, 3, 6, 7 sit on quadrants 2, 3 (rows >= 64, never stored) and only join the final
// barriers.  (Round 1 had 6 warps with 2 working epilogue warps of 32 units each: the gate math
// of a step then took ~1.0 us; split over 4 warps it halves, tools/latency_bench.cu.)
constexpr int KTHREADS = 320;
constexpr int KEPI = 4;     // working epilogue warps
constexpr int XSTAGES = 3;
constexpr int X_BYTES = KB * KBK * 2;  // 8 KiB: 64 rows x 64 units (SW128)

// Per-CTA slice width KU (hidden units per CTA; the cluster has H / KU CTAs): 32 (8-CTA clusters
// at H = 256) or 16 (16-CTA clusters: half the MMA and gate math per step — the critical path —
// for the same DSMEM send volume per CTA).
template <int KU>
struct KC {
    static constexpr int KN = 4 * KU;                         // UMMA N (i | f | o | ĝ)
    static constexpr int KEU = KU / 2;                        // units per epilogue thread
    static constexpr int GATE_BYTES = KU * KBK * 2;           // one gate's KU units x 64 K
    static constexpr int WCHUNK = 4 * GATE_BYTES;             // the 4 gates of one K chunk
    static constexpr int SLICE_BYTES = KB * KU * 2;           // one CTA's h slice (KU/8 k-groups x 64 rows)
    static constexpr uint32_t WLAYOUT = KU == 32 ? 4u : 6u;   // SWIZZLE_64B / SWIZZLE_32B (MN-major)
    static constexpr uint32_t IDESC = make_idesc_bf16_f32(KROWS, KN, false, true);
    static constexpr int TMEM_COLS = 2 * KN < 32 ? 32 : 2 * KN;
};

struct KMaps {
    CUtensorMap x, h, W, U;
};

struct KLayout {  // byte offsets into the 1024-aligned dynamic shared memory
    int rec0, rec1, xring, w, bars, bias, total;
};

template <int KU>
__host__ __device__ constexpr KLayout klayout(int H) {
    KLayout L{};
    const int rec = (H / 8) * 1024;  // H/8 k-groups x 1 KiB
    L.rec0 = 0;
    L.rec1 = rec;
    L.xring = 2 * rec;
    L.w = L.xring + XSTAGES * X_BYTES;
    L.bars = L.w + 2 * (H / KBK) * KC<KU>::WCHUNK;
    L.bias = L.bars + 256;
    L.total = L.bias + 4 * KU * 4;
    return L;
}

__device__ __forceinline__ uint32_t kpack(float lo, float hi) {
    __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
    return *reinterpret_cast<uint32_t*>(&v);
}

// 16-byte asynchronous store into a cluster peer's shared memory; complete_tx(16) on its mbarrier.
__device__ __forceinline__ void st_async_v4(uint32_t dst_cluster, uint4 v, uint32_t mbar_cluster) {
    asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %2, %3, %4}, [%5];" ::"r"(
                     dst_cluster),
                 "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "r"(mbar_cluster)
                 : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

template <int KU>
__global__ void __launch_bounds__(KTHREADS, 1)
wavefront_cluster_kernel(const __grid_constant__ Problem P, const __grid_constant__ Tensors T,
                         const __grid_constant__ KMaps M) {
    using C = KC<KU>;
    constexpr int KN = C::KN, KEU = C::KEU, GATE_BYTES = C::GATE_BYTES, WCHUNK = C::WCHUNK;
    constexpr int SLICE_BYTES = C::SLICE_BYTES;
    constexpr uint32_t IDESC = C::IDESC;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    uint8_t* smem = smem_raw + pad;
    const KLayout L = klayout<KU>(P.H);
    const int KCH = P.H / KBK;           // K chunks per half
    const int CS = P.H / KU;             // CTAs per layer = cluster size
    uint8_t* rec[2] = {smem + L.rec0, smem + L.rec1};
    uint8_t* xring = smem + L.xring;
    uint8_t* sW = smem + L.w;
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + L.bars);
    uint64_t* xfull = bars;                       // [XSTAGES]
    uint64_t* xempty = bars + XSTAGES;            // [XSTAGES]
    uint64_t* tfull = bars + 2 * XSTAGES;         // [2]
    uint64_t* tempty = tfull + 2;                 // [2]
    uint64_t* hfull = tempty + 2;                 // [2] recurrent buffers (DSMEM complete_tx)
    uint64_t* wbar = hfull + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(wbar + 1);
    float* sbias = reinterpret_cast<float*>(smem + L.bias);  // [4][KU]

    const uint32_t j = cluster_ctarank();        // unit slab inside the layer
    const int d = blockIdx.x / CS;               // layer = cluster
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rec_bytes = (uint32_t)KB * P.H * 2;  // one full h_{d,t} (all CS slices)

    if (threadIdx.x == 0) {
        for (int s = 0; s < XSTAGES; ++s) {
            mbar_init(&xfull[s], 1);
            mbar_init(&xempty[s], 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&tfull[a], 1);
            mbar_init(&tempty[a], KEPI);  // the working epilogue warps
            mbar_init(&hfull[a], 1);
        }
        mbar_init(wbar, 1);
        fence_mbarrier_init();
        // arm both recurrent buffers for their first phase (h_0 → rec0, h_1 → rec1) before any
        // peer can send: the cluster barrier below orders this before every peer's first copy
        mbar_arrive_expect_tx(&hfull[0], rec_bytes);
        mbar_arrive_expect_tx(&hfull[1], rec_bytes);
    }
    if (threadIdx.x >= 64 && threadIdx.x < 64 + 4 * KU) {  // (4·KU <= 128 <= 256 threads past warp 1)
        const int e = threadIdx.x - 64;
        sbias[e] = T.b[(long long)d * 4 * P.H + (e / KU) * P.H + (int)j * KU + e % KU];
    }
    if (warp == 1) tmem_alloc(tmem_slot, C::TMEM_COLS);
    tc_fence_before();
    __syncthreads();
    cluster_sync();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {
            // ---- the slab's weights → shared memory, once for the whole sequence -------------
            const uint64_t pol_keep = policy_evict_last();
            const uint64_t pol_act = policy_evict_normal();
            mbar_arrive_expect_tx(wbar, 2 * KCH * WCHUNK);
            for (int c = 0; c < 2 * KCH; ++c)
                tma_load_4d_hint_addr<1>(smem_u32(sW + c * WCHUNK), c < KCH ? &M.W : &M.U, smem_u32(wbar),
                                         (int)j * KU, (c % KCH) * KBK, 0, d, pol_keep);
            // ---- per step: the input half (x or the layer below) -----------------------------
            int stage = 0;
            uint32_t phase = 0;
            for (int t = 0; t < P.L0; ++t) {
                if (d > 0) {  // depth edge: layer d-1's cell (d-1, t), all CS slices
                    wait_flag_geq(T.flags + cell_lin(P, d - 1, t, 0), CS);
                    fence_proxy_async_global();
                }
                for (int kc = 0; kc < KCH; ++kc) {
                    mbar_wait(&xempty[stage], phase ^ 1);
                    mbar_arrive_expect_tx(&xfull[stage], X_BYTES);
                    const uint32_t dst = smem_u32(xring + stage * X_BYTES);
                    const uint32_t bar = smem_u32(&xfull[stage]);
                    if (d == 0)
                        tma_load_3d_hint_addr<1>(dst, &M.x, bar, kc * KBK, t, 0, pol_act);
                    else
                        tma_load_2d_hint_addr<1>(dst, &M.h, bar, 0,
                                                 (int)hb_row(P, h_row(P, d - 1, t, 0, 0), kc, 0), pol_act);
                    if (++stage == XSTAGES) {
                        stage = 0;
                        phase ^= 1;
                    }
                }
            }
        }
    } else if (warp == 1) {
        // ---- MMA issuer (whole warp; warp-uniform waits keep descriptors uniform) ------------
        mbar_wait_warp(wbar, 0);
        tc_fence_after();
        const uint64_t xdesc0 = make_sdesc(smem_u32(xring), 16, 1024);                 // SW128 K-major
        const uint64_t rdesc[2] = {make_sdesc(smem_u32(rec[0]), 1024, 128, 0),         // no swizzle
                                   make_sdesc(smem_u32(rec[1]), 1024, 128, 0)};
        const uint64_t bdesc0 = make_sdesc(smem_u32(sW), GATE_BYTES, 8 * KU * 2, C::WLAYOUT);  // MN-major
        int stage = 0, acc = 0;
        uint32_t phase = 0, acc_phase = 0;
        for (int t = 0; t < P.L0; ++t) {
            mbar_wait_warp(&tempty[acc], acc_phase ^ 1);
            tc_fence_after();
            const uint32_t d_tmem = tmem_base + (uint32_t)(acc * KN);
            // input half first: it arrives early (the layer below runs ahead)
            for (int kc = 0; kc < KCH; ++kc) {
                mbar_wait_warp(&xfull[stage], phase);
                if (kc == 0 && lane == 0) FT_CEV(t, 5);
                tc_fence_after();
                if (elect_one()) {
                    const uint64_t ad = xdesc0 + (uint64_t)((stage * X_BYTES) >> 4);
                    const uint64_t bd = bdesc0 + (uint64_t)((kc * WCHUNK) >> 4);
#pragma unroll
                    for (int kk = 0; kk < KBK / 16; ++kk)
                        umma_f16(d_tmem, ad + (uint64_t)((kk * 32) >> 4), bd + (uint64_t)((kk * 16 * KU * 2) >> 4),
                                 IDESC, (kc | kk) != 0);
                    umma_commit(&xempty[stage]);
                }
                __syncwarp();
                if (++stage == XSTAGES) {
                    stage = 0;
                    phase ^= 1;
                }
            }
            if (t > 0) {  // time edge: h_{d,t-1} from every cluster CTA, through DSMEM
                const int p = (t - 1) & 1;
                mbar_wait_warp(&hfull[p], (uint32_t)((t - 1) >> 1) & 1u);
                if (lane == 0) FT_CEV(t, 0);
                fence_proxy_async_smem();  // peers' st.async data → this CTA's tensor-core reads
                tc_fence_after();
                if (elect_one()) {
                    // re-arm this buffer for h_{t+1}: its senders first need our h_t, which we
                    // send only after these MMAs completed — so the next phase cannot start early
                    mbar_arrive_expect_tx(&hfull[p], rec_bytes);
                    for (int kc = 0; kc < KCH; ++kc) {
                        const uint64_t bd = bdesc0 + (uint64_t)(((KCH + kc) * WCHUNK) >> 4);
#pragma unroll
                        for (int kk = 0; kk < KBK / 16; ++kk)
                            umma_f16(d_tmem, rdesc[p] + (uint64_t)(((kc * 8 + kk * 2) * 1024) >> 4),
                                     bd + (uint64_t)((kk * 16 * KU * 2) >> 4), IDESC, 1u);
                    }
                }
                __syncwarp();
            }
            if (elect_one()) umma_commit(&tfull[acc]);
            if (lane == 0) FT_CEV(t, 1);
            __syncwarp();
            acc ^= 1;
            if (acc == 0) acc_phase ^= 1;
        }
    } else if (warp >= 4 && (warp & 3) < 2) {
        // ---- epilogue: warps of TMEM lane quadrants 0 and 1 (rows 0..63), KEU units each; c in
        //      registers.  half = which 16 units of the CTA's 32-unit slice this warp owns.
        const int q = warp & 3, row = q * 32 + lane, half = warp >= 8;
        const bool valid = row < P.B;
        const int n0 = (int)j * KU + half * KEU;
        const bool sender = (warp == 4 && lane == 0);
        float creg[KEU];
#pragma unroll
        for (int u = 0; u < KEU; ++u) creg[u] = 0.f;
        __nv_bfloat16* hb = (__nv_bfloat16*)T.hb;
        __nv_bfloat16* h_all = (__nv_bfloat16*)T.h_all;
        int acc = 0;
        uint32_t acc_phase = 0;
        for (int t = 0; t < P.L0; ++t) {
            mbar_wait(&tfull[acc], acc_phase);
            if (sender) FT_CEV(t, 2);
            if (sender && j == 0) FT_LEV(d, t);
            tc_fence_after();
            const uint32_t tbase = tmem_base + (uint32_t)(acc * KN) + ((uint32_t)(q * 32) << 16) + half * KEU;
            uint32_t hp[KEU / 2];
            {
                float zi[KEU], zf[KEU], zo[KEU], zg[KEU];
                tmem_ld_32x32b<KEU>(tbase + 0 * KU, zi);
                tmem_ld_32x32b<KEU>(tbase + 1 * KU, zf);
                tmem_ld_32x32b<KEU>(tbase + 2 * KU, zo);
                tmem_ld_32x32b<KEU>(tbase + 3 * KU, zg);
                tmem_wait_ld();
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&tempty[acc]);
                const int ub = half * KEU;
                // (1) the time edge first, pipelined with the math: as soon as a k-group of 8 units
                //     is done, every thread st.async's its row of it (16 B) straight from registers
                //     into every cluster CTA's buffer t & 1, each store carrying complete_tx(16) to
                //     that CTA's hfull[t & 1] (no staging, no barrier); the next k-group's math
                //     overlaps those stores in flight
                const uint32_t dst_local = smem_u32(rec[t & 1]) + j * SLICE_BYTES +
                                           (uint32_t)half * (KEU / 8) * 1024u + (uint32_t)row * 16u;
                const uint32_t bar_local = smem_u32(&hfull[t & 1]);
#pragma unroll
                for (int g = 0; g < KEU / 8; ++g) {
#pragma unroll
                    for (int v = 8 * g; v < 8 * g + 8; ++v) {
                        const float ig = sigmoid_approx(zi[v] + sbias[0 * KU + ub + v]);
                        const float fg = sigmoid_approx(zf[v] + sbias[1 * KU + ub + v]);
                        const float og = sigmoid_approx(zo[v] + sbias[2 * KU + ub + v]);
                        const float gh = tanh_approx(zg[v] + sbias[3 * KU + ub + v]);
                        creg[v] = fmaf(fg, creg[v], ig * gh);
                        zi[v] = og * tanh_approx(creg[v]);  // h
                    }
#pragma unroll
                    for (int v = 4 * g; v < 4 * g + 4; ++v) hp[v] = kpack(zi[2 * v], zi[2 * v + 1]);
                    if (t + 1 < P.L0) {
                        const uint4 val = make_uint4(hp[4 * g], hp[4 * g + 1], hp[4 * g + 2], hp[4 * g + 3]);
                        for (int r = 0; r < CS; ++r)
                            st_async_v4(mapa_shared(dst_local, (uint32_t)r) + g * 1024u, val,
                                        mapa_shared(bar_local, (uint32_t)r));
                    }
                }
                if (sender) FT_CEV(t, 3);
            }
            if (sender) FT_CEV(t, 4);
            // (2) the depth edge: h into the blocked SSA buffer, then one cumulative release
            const Cell cell{d + t, d, t, 0};
            if (valid) {
                uint4* dst = reinterpret_cast<uint4*>(hb + hb_row(P, h_row(P, d, t, 0, 0), n0 / 64, row) * 64 + (n0 % 64));
#pragma unroll
                for (int w = 0; w < KEU / 8; ++w)
                    __stcg(dst + w, make_uint4(hp[4 * w], hp[4 * w + 1], hp[4 * w + 2], hp[4 * w + 3]));
            }
            named_bar_sync(1, KEPI * 32);
            if (sender && d + 1 < P.D) red_release_gpu_add(T.flags + cell_lin(P, d, t, 0), 1);
            // (3) outputs nobody inside the nest reads
            if (valid) {
                const long long hi = h_all_index(P, cell, 0, row, n0);
                if (h_all) {
                    uint4* dh = reinterpret_cast<uint4*>(h_all + hi);
#pragma unroll
                    for (int w = 0; w < KEU / 8; ++w)
                        dh[w] = make_uint4(hp[4 * w], hp[4 * w + 1], hp[4 * w + 2], hp[4 * w + 3]);
                }
                if (T.c_all) {
                    float4* dc = reinterpret_cast<float4*>(T.c_all + hi);
#pragma unroll
                    for (int w = 0; w < KEU / 4; ++w)
                        dc[w] = make_float4(creg[4 * w], creg[4 * w + 1], creg[4 * w + 2], creg[4 * w + 3]);
                }
                if (d == P.D - 1) {
                    uint4* dy = reinterpret_cast<uint4*>((__nv_bfloat16*)T.y + y_index(P, cell, 0, row, n0));
#pragma unroll
                    for (int w = 0; w < KEU / 8; ++w)
                        dy[w] = make_uint4(hp[4 * w], hp[4 * w + 1], hp[4 * w + 2], hp[4 * w + 3]);
                }
                if (t == P.L0 - 1) {
                    const long long ni = hn_index(P, cell, 0, row, n0);
                    uint4* dn = reinterpret_cast<uint4*>((__nv_bfloat16*)T.h_n + ni);
#pragma unroll
                    for (int w = 0; w < KEU / 8; ++w)
                        dn[w] = make_uint4(hp[4 * w], hp[4 * w + 1], hp[4 * w + 2], hp[4 * w + 3]);
                    float4* dc = reinterpret_cast<float4*>(T.c_n + ni);
#pragma unroll
                    for (int w = 0; w < KEU / 4; ++w)
                        dc[w] = make_float4(creg[4 * w], creg[4 * w + 1], creg[4 * w + 2], creg[4 * w + 3]);
                }
            }
            acc ^= 1;
            if (acc == 0) acc_phase ^= 1;
        }
    }
    tc_fence_before();
    __syncthreads();
    cluster_sync();  // no CTA leaves while a peer may still copy into its shared memory
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc(tmem_base, C::TMEM_COLS);
    }
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

bool kenc(EncodeTiledFn enc, CUtensorMap* m, int rank, const void* base, const cuuint64_t* dims,
          const cuuint64_t* strides, const cuuint32_t* box, CUtensorMapSwizzle sw, std::string* err) {
    const cuuint32_t es[4] = {1, 1, 1, 1};
    CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, rank, const_cast<void*>(base), dims, strides, box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
        if (err) *err = "cuTensorMapEncodeTiled (cluster) failed: " + std::to_string((int)r);
        return false;
    }
    return true;
}

template <int KU>
size_t cluster_smem(int H) { return (size_t)klayout<KU>(H).total + 1024; }

// Can the D clusters of H / KU CTAs (one per SM) all be co-resident?  (16-CTA clusters need the
// non-portable cluster size opt-in.)
template <int KU>
bool cluster_fits(const Problem& p) {
    const int cs = p.H / KU;
    if (cs > 16 || cluster_smem<KU>(p.H) > 227 * 1024) return false;
    if (cs > 8 && cudaFuncSetAttribute(wavefront_cluster_kernel<KU>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) !=
                      cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (cudaFuncSetAttribute(wavefront_cluster_kernel<KU>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)cluster_smem<KU>(p.H)) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(p.D * cs));
    cfg.blockDim = dim3(KTHREADS);
    cfg.dynamicSmemBytes = cluster_smem<KU>(p.H);
    cudaLaunchAttribute a[1];
    a[0].id = cudaLaunchAttributeClusterDimension;
    a[0].val.clusterDim.x = cs;
    a[0].val.clusterDim.y = 1;
    a[0].val.clusterDim.z = 1;
    cfg.attrs = a;
    cfg.numAttrs = 1;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, wavefront_cluster_kernel<KU>, &cfg) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return n >= p.D;
}

// Slice width: 16 units (clusters of H/16 CTAs) when they fit, else 32; 0 = the kernel does not
// apply.  FT_CLUSTER_UNITS=32|16 forces one (A/B).
int cluster_units(const Problem& p) {
    if (p.kind != KIND_SEQ || p.cell != CELL_LSTM || p.B > KB || (p.H != 128 && p.H != 256)) return 0;
    for (int d = 0; d < p.D; ++d)
        if (p.dil[d] != 1) return 0;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return 0;
    const char* e = getenv("FT_CLUSTER_UNITS");
    const int want = e ? atoi(e) : 0;
    if (want != 32 && cluster_fits<16>(p)) return 16;
    if (want != 16 && cluster_fits<32>(p)) return 32;
    return 0;
}

template <int KU>
cudaError_t launch_cluster_t(const Problem& p, const Tensors& t, cudaStream_t s, std::string* err) {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q = cudaDriverEntryPointSymbolNotFound;
    cudaError_t e = cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &ptr, 12000, cudaEnableDefault, &q);
    if (e != cudaSuccess || !ptr) {
        if (err) *err = "cuTensorMapEncodeTiled not available";
        return cudaErrorNotSupported;
    }
    EncodeTiledFn enc = reinterpret_cast<EncodeTiledFn>(ptr);
    KMaps M;
    const int H = p.H;
    {  // x [B][T][H]: a (64 units, 1 step, 64 rows) box
        const cuuint64_t dims[3] = {(cuuint64_t)H, (cuuint64_t)p.L0, (cuuint64_t)p.B};
        const cuuint64_t st[2] = {(cuuint64_t)H * 2, (cuuint64_t)p.L0 * H * 2};
        const cuuint32_t box[3] = {KBK, 1, KB};
        if (!kenc(enc, &M.x, 3, t.x, dims, st, box, CU_TENSOR_MAP_SWIZZLE_128B, err)) return cudaErrorInvalidValue;
    }
    {  // blocked SSA buffer hb: a (64 units, 64 rows) box
        const cuuint64_t dims[2] = {64, (cuuint64_t)hb_rows_total(p)};
        const cuuint64_t st[1] = {128};
        const cuuint32_t box[2] = {KBK, KB};
        if (!kenc(enc, &M.h, 2, t.hb, dims, st, box, CU_TENSOR_MAP_SWIZZLE_128B, err)) return cudaErrorInvalidValue;
    }
    {  // weights (n, k, gate, layer): (KU units, 64 K, 4 gates, 1) boxes, 64- / 32-byte swizzle
        const cuuint64_t dims[4] = {(cuuint64_t)H, (cuuint64_t)H, 4, (cuuint64_t)p.D};
        const cuuint64_t st[3] = {(cuuint64_t)H * 2, (cuuint64_t)H * H * 2, (cuuint64_t)4 * H * H * 2};
        const cuuint32_t box[4] = {KU, KBK, 4, 1};
        const CUtensorMapSwizzle sw = KU == 32 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
        if (!kenc(enc, &M.W, 4, t.W, dims, st, box, sw, err)) return cudaErrorInvalidValue;
        if (!kenc(enc, &M.U, 4, t.U, dims, st, box, sw, err)) return cudaErrorInvalidValue;
    }
    const size_t smem = cluster_smem<KU>(H);
    e = cudaFuncSetAttribute(wavefront_cluster_kernel<KU>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess && H / KU > 8)
        e = cudaFuncSetAttribute(wavefront_cluster_kernel<KU>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) {
        if (err) *err = std::string("cluster launch setup: ") + cudaGetErrorString(e);
        return e;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(p.D * (H / KU)));
    cfg.blockDim = dim3(KTHREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;  // one cluster per layer
    attr[0].val.clusterDim.x = H / KU;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    int coop = 0;
    e = launch_cluster_persistent(cfg, attr, 1, &coop, wavefront_cluster_kernel<KU>, p, t, M);
    if (e == cudaSuccess)
        set_last_launch("wavefront_cluster_kernel<" + std::to_string(KU) + "> grid=" + std::to_string(p.D * (H / KU)) +
                        " cluster=" + std::to_string(H / KU) + " cooperative=" + std::to_string(coop));
    if (e != cudaSuccess && err) *err = std::string("cluster launch: ") + cudaGetErrorString(e);
    return e;
}

}  // namespace

// The DSMEM-exchange kernel applies when: stacked LSTM (every dilation 1), batch <= 64, H in
// {128, 256}, bf16, and the D clusters of H/KU CTAs (one CTA per SM) can all be co-resident.
bool cluster_kernel_applies(const Problem& p) { return cluster_units(p) != 0; }

cudaError_t launch_wavefront_cluster(const Problem& p, const Tensors& t, cudaStream_t s, std::string* err) {
    const int ku = cluster_units(p);
    if (ku == 16) return launch_cluster_t<16>(p, t, s, err);
    if (ku == 32) return launch_cluster_t<32>(p, t, s, err);
    if (err) *err = "cluster kernel does not apply";
    return cudaErrorInvalidConfiguration;
}

}  // namespace ft
