// wavefront_resident.cu — a5 "weights resident across time": the sm_100a wavefront for stacked
// LSTMs whose whole weight set fits in the SMs' shared memory (e.g. C2: 8 MiB over 128 SMs).
//
// The paper's reuse analysis (null space of the weight access e14 spans batch and hidden,
// L345–L349) says one load of W_d / U_d can serve every (batch, time) iteration of layer d.  Here
// that reuse is taken literally: CTA (d, n) owns the slab W[d][:, gates, n*BNU : (n+1)*BNU] and
// U[d][...] for the WHOLE sequence — TMA-loaded into shared memory once, consumed by every time
// step's tcgen05.mma straight from SMEM — and keeps its cell state c in registers across time
// (the same threads own the same (row, unit) pairs at every step).  Per step only the activation
// K-chunks stream in (TMA, 16 KiB each).  The wavefront emerges from the per-(cell) readiness
// counters: layer d runs step t as soon as layer d-1 finished t and layer d finished t-1 (Table 4
// dependence vectors; π = d + t, L341/L349).
//
// Tile: M = 128 batch rows (batch <= 128), N = 4 gates x BNU units (BNU = 16 → N = 64 with a
// 32-byte-swizzled MN-major weight operand, BNU = 32 → N = 128 with 64-byte swizzle), K = 64 per
// chunk.  Warps: 0 TMA producer, 1 MMA issuer, 2–5 epilogue (one batch row per thread).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <string>

#include "ft_internal.h"
#include "ft_sm100.cuh"

namespace ft {
namespace {

using namespace sm100;

constexpr int RROWS = 128;
constexpr int RBK = 64;
constexpr int RTHREADS = 192;

template <int BNUR>
struct RCfg {
    static constexpr int N = 4 * BNUR;                         // UMMA N
    static constexpr int SW = BNUR * 2;                        // bytes per weight smem row (swizzle span)
    static constexpr uint32_t LAYOUT = BNUR == 16 ? 6u : 4u;   // SWIZZLE_32B / SWIZZLE_64B
    static constexpr int GATE_BYTES = BNUR * RBK * 2;          // one gate atom column of a K chunk
    static constexpr int WCHUNK = 4 * GATE_BYTES;              // one K chunk of the weight slab
    static constexpr int A_BYTES = RROWS * RBK * 2;            // 16 KiB
    static constexpr int STAGES = 4;
    static constexpr int TMEM_COLS = 2 * N < 32 ? 32 : 2 * N;
    static constexpr uint32_t IDESC = make_idesc_bf16_f32(RROWS, N, false, true);
};

struct RMaps {
    CUtensorMap x, h, W, U;
};

__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
    __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
    return *reinterpret_cast<uint32_t*>(&v);
}

// shared-memory layout: weight slab | A ring | barriers + TMEM slot (256 B) | bias [4][BNUR]
template <int BNUR>
__host__ __device__ constexpr int resident_bias_off(int H) {
    return 2 * (H / RBK) * RCfg<BNUR>::WCHUNK + RCfg<BNUR>::STAGES * RCfg<BNUR>::A_BYTES + 256;
}

template <int BNUR>
__global__ void __launch_bounds__(RTHREADS, 1)
wavefront_resident_kernel(const __grid_constant__ Problem P, const __grid_constant__ Tensors T,
                          const __grid_constant__ RMaps M) {
    using C = RCfg<BNUR>;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    uint8_t* smem = smem_raw + pad;
    const int KCH = P.H / RBK;                      // K chunks per half (input or recurrent)
    uint8_t* sW = smem;                             // 2*KCH resident weight chunks
    uint8_t* sA = smem + 2 * KCH * C::WCHUNK;       // A ring
    uint64_t* bars = reinterpret_cast<uint64_t*>(sA + C::STAGES * C::A_BYTES);
    uint64_t* full = bars;
    uint64_t* empty = bars + C::STAGES;
    uint64_t* tfull = bars + 2 * C::STAGES;
    uint64_t* tempty = tfull + 2;
    uint64_t* wbar = tempty + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(wbar + 1);
    float* sbias = reinterpret_cast<float*>(smem_raw + pad + resident_bias_off<BNUR>(P.H));  // [4][BNUR]

    const int NTR = P.H / BNUR;
    const int d = blockIdx.x / NTR, n = blockIdx.x % NTR;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < C::STAGES; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&tfull[a], 1);
            mbar_init(&tempty[a], 4);
        }
        mbar_init(wbar, 1);
        fence_mbarrier_init();
    }
    if (warp == 1) tmem_alloc(tmem_slot, C::TMEM_COLS);
    // the slab's bias → shared memory once: the per-step acquires invalidate L1 (CCTL.IVALL), so
    // global bias loads in the epilogue would go to L2 on the critical path every step
    if (threadIdx.x >= 64 && threadIdx.x < 64 + 4 * BNUR) {
        const int e = threadIdx.x - 64;
        sbias[e] = T.b[(long long)(blockIdx.x / (P.H / BNUR)) * 4 * P.H + (e / BNUR) * P.H +
                       (blockIdx.x % (P.H / BNUR)) * BNUR + e % BNUR];
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    const int target = NTR;

    if (warp == 0) {
        if (lane == 0) {
            // ---- the layer's weight slab → shared memory, once for the whole sequence -------
            const uint64_t pol_keep = policy_evict_last();
            const uint64_t pol_act = policy_evict_normal();
            mbar_arrive_expect_tx(wbar, 2 * KCH * C::WCHUNK);
            for (int c = 0; c < 2 * KCH; ++c)
                tma_load_4d_hint_addr<1>(smem_u32(sW + c * C::WCHUNK), c < KCH ? &M.W : &M.U,
                                         smem_u32(wbar), n * BNUR, (c % KCH) * RBK, 0, d, pol_keep);
            // ---- per time step: the activation K-chunks ------------------------------------
            int stage = 0;
            uint32_t phase = 0;
            for (int t = 0; t < P.L0; ++t) {
                const int nch = (t > 0 ? 2 : 1) * KCH;
                for (int c = 0; c < nch; ++c) {
                    // acquire each half's producer just before its first chunk: the input half
                    // (layer below / x) streams in while the recurrent producer still runs
                    if (c == 0 && d > 0) {
                        wait_flag_geq(T.flags + cell_lin(P, d - 1, t, 0), target);
                        fence_proxy_async_global();
                    }
                    if (c == KCH) {
                        wait_flag_geq(T.flags + cell_lin(P, d, t - 1, 0), target);
                        fence_proxy_async_global();
                    }
                    mbar_wait(&empty[stage], phase ^ 1);
                    mbar_arrive_expect_tx(&full[stage], C::A_BYTES);
                    const uint32_t dst = smem_u32(sA + stage * C::A_BYTES);
                    const uint32_t bar = smem_u32(&full[stage]);
                    const int kc = c % KCH;
                    if (c < KCH && d == 0)
                        tma_load_3d_hint_addr<1>(dst, &M.x, bar, kc * RBK, t, 0, pol_act);
                    else
                        tma_load_2d_hint_addr<1>(dst, &M.h, bar, 0,
                                                 (int)hb_row(P, c < KCH ? h_row(P, d - 1, t, 0, 0)
                                                                        : h_row(P, d, t - 1, 0, 0),
                                                             kc, 0),
                                                 pol_act);
                    if (++stage == C::STAGES) {
                        stage = 0;
                        phase ^= 1;
                    }
                }
            }
        }
    } else if (warp == 1) {
        {  // the whole warp (warp-uniform waits keep the MMA descriptors in uniform registers)
            mbar_wait_warp(wbar, 0);
            tc_fence_after();
            const uint64_t adesc0 = make_sdesc(smem_u32(sA), 16, 1024);
            // weights: MN-major, BNU-wide swizzle atoms; gate atoms GATE_BYTES apart (LBO),
            // 8-k-row groups 8*SW apart (SBO); K step of 16 rows = 16*SW bytes.
            const uint64_t bdesc0 = make_sdesc(smem_u32(sW), C::GATE_BYTES, 8 * C::SW, C::LAYOUT);
            int stage = 0, acc = 0;
            uint32_t phase = 0, acc_phase = 0;
            for (int t = 0; t < P.L0; ++t) {
                mbar_wait_warp(&tempty[acc], acc_phase ^ 1);
                tc_fence_after();
                const uint32_t d_tmem = tmem_base + (uint32_t)(acc * C::N);
                const int nch = (t > 0 ? 2 : 1) * KCH;
                for (int c = 0; c < nch; ++c) {
                    mbar_wait_warp(&full[stage], phase);
                    tc_fence_after();
                    if (elect_one()) {
                        const uint64_t ad = adesc0 + (uint64_t)((stage * C::A_BYTES) >> 4);
                        const uint64_t bd = bdesc0 + (uint64_t)((c * C::WCHUNK) >> 4);
#pragma unroll
                        for (int kk = 0; kk < RBK / 16; ++kk)
                            umma_f16(d_tmem, ad + (uint64_t)((kk * 32) >> 4),
                                     bd + (uint64_t)((kk * 16 * C::SW) >> 4), C::IDESC, (c | kk) != 0);
                        umma_commit(&empty[stage]);
                    }
                    __syncwarp();
                    if (++stage == C::STAGES) {
                        stage = 0;
                        phase ^= 1;
                    }
                }
                if (elect_one()) umma_commit(&tfull[acc]);
                __syncwarp();
                acc ^= 1;
                if (acc == 0) acc_phase ^= 1;
            }
        }
    } else {
        // ---- epilogue: one batch row per thread, all BNU units; c lives in registers --------
        const int q = warp & 3, row = q * 32 + lane;
        const bool valid = row < P.B;
        const int n0 = n * BNUR;
        float creg[BNUR];
#pragma unroll
        for (int u = 0; u < BNUR; ++u) creg[u] = 0.f;
        __nv_bfloat16* hb = (__nv_bfloat16*)T.hb;
        __nv_bfloat16* h_all = (__nv_bfloat16*)T.h_all;
        int acc = 0;
        uint32_t acc_phase = 0;
        for (int t = 0; t < P.L0; ++t) {
            mbar_wait(&tfull[acc], acc_phase);
            tc_fence_after();
            const uint32_t tbase = tmem_base + (uint32_t)(acc * C::N) + ((uint32_t)(q * 32) << 16);
            uint32_t hp[BNUR / 2];
#pragma unroll
            for (int u0 = 0; u0 < BNUR; u0 += 16) {
                float zi[16], zf[16], zo[16], zg[16];
                tmem_ld_32x32b_x16(tbase + 0 * BNUR + u0, zi);
                tmem_ld_32x32b_x16(tbase + 1 * BNUR + u0, zf);
                tmem_ld_32x32b_x16(tbase + 2 * BNUR + u0, zo);
                tmem_ld_32x32b_x16(tbase + 3 * BNUR + u0, zg);
                tmem_wait_ld();
                if (u0 + 16 == BNUR) {
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&tempty[acc]);
                }
#pragma unroll
                for (int v = 0; v < 16; ++v) {
                    const float ig = sigmoid_approx(zi[v] + sbias[0 * BNUR + u0 + v]);
                    const float fg = sigmoid_approx(zf[v] + sbias[1 * BNUR + u0 + v]);
                    const float og = sigmoid_approx(zo[v] + sbias[2 * BNUR + u0 + v]);
                    const float gh = tanh_approx(zg[v] + sbias[3 * BNUR + u0 + v]);
                    creg[u0 + v] = fmaf(fg, creg[u0 + v], ig * gh);
                    zi[v] = og * tanh_approx(creg[u0 + v]);  // h
                }
#pragma unroll
                for (int v = 0; v < 8; ++v) hp[u0 / 2 + v] = pack2(zi[2 * v], zi[2 * v + 1]);
            }
            const Cell cell{d + t, d, t, 0};
            if (valid) {
                uint4* dst = reinterpret_cast<uint4*>(hb + hb_row(P, h_row(P, d, t, 0, 0), n0 / 64, row) * 64 + (n0 % 64));
#pragma unroll
                for (int w = 0; w < BNUR / 8; ++w)
                    __stcg(dst + w, make_uint4(hp[4 * w], hp[4 * w + 1], hp[4 * w + 2], hp[4 * w + 3]));
            }
            named_bar_sync(1, 128);  // every epilogue thread's h stores, then ONE cumulative release
            if (threadIdx.x == 64) red_release_gpu_add(T.flags + cell_lin(P, d, t, 0), 1);
            if (valid) {  // outputs nobody inside the nest reads
                const long long hi = h_all_index(P, cell, 0, row, n0);
                if (h_all) {
                    uint4* dh = reinterpret_cast<uint4*>(h_all + hi);
#pragma unroll
                    for (int w = 0; w < BNUR / 8; ++w)
                        dh[w] = make_uint4(hp[4 * w], hp[4 * w + 1], hp[4 * w + 2], hp[4 * w + 3]);
                }
                if (T.c_all) {
                    float4* dc = reinterpret_cast<float4*>(T.c_all + hi);
#pragma unroll
                    for (int w = 0; w < BNUR / 4; ++w)
                        dc[w] = make_float4(creg[4 * w], creg[4 * w + 1], creg[4 * w + 2], creg[4 * w + 3]);
                }
                if (d == P.D - 1) {
                    uint4* dy = reinterpret_cast<uint4*>((__nv_bfloat16*)T.y + y_index(P, cell, 0, row, n0));
#pragma unroll
                    for (int w = 0; w < BNUR / 8; ++w)
                        dy[w] = make_uint4(hp[4 * w], hp[4 * w + 1], hp[4 * w + 2], hp[4 * w + 3]);
                }
                if (t == P.L0 - 1) {
                    const long long ni = hn_index(P, cell, 0, row, n0);
                    uint4* dn = reinterpret_cast<uint4*>((__nv_bfloat16*)T.h_n + ni);
#pragma unroll
                    for (int w = 0; w < BNUR / 8; ++w)
                        dn[w] = make_uint4(hp[4 * w], hp[4 * w + 1], hp[4 * w + 2], hp[4 * w + 3]);
                    float4* dc = reinterpret_cast<float4*>(T.c_n + ni);
#pragma unroll
                    for (int w = 0; w < BNUR / 4; ++w)
                        dc[w] = make_float4(creg[4 * w], creg[4 * w + 1], creg[4 * w + 2], creg[4 * w + 3]);
                }
            }
            acc ^= 1;
            if (acc == 0) acc_phase ^= 1;
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc(tmem_base, C::TMEM_COLS);
    }
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

bool enc_map(EncodeTiledFn enc, CUtensorMap* m, int rank, const void* base, const cuuint64_t* dims,
             const cuuint64_t* strides, const cuuint32_t* box, CUtensorMapSwizzle sw, std::string* err) {
    const cuuint32_t es[4] = {1, 1, 1, 1};
    CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, rank, const_cast<void*>(base), dims, strides,
                     box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
        if (err) *err = "cuTensorMapEncodeTiled (resident) failed: " + std::to_string((int)r);
        return false;
    }
    return true;
}

template <int BNUR>
size_t resident_smem(int H) {
    using C = RCfg<BNUR>;
    return (size_t)2 * (H / RBK) * C::WCHUNK + C::STAGES * C::A_BYTES + 256 + 4 * BNUR * 4 + 1024;
}

template <int BNUR>
cudaError_t launch_resident_t(const Problem& p, const Tensors& t, cudaStream_t s, std::string* err) {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q = cudaDriverEntryPointSymbolNotFound;
    cudaError_t e = cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &ptr, 12000,
                                                     cudaEnableDefault, &q);
    if (e != cudaSuccess || !ptr) {
        if (err) *err = "cuTensorMapEncodeTiled not available";
        return cudaErrorNotSupported;
    }
    EncodeTiledFn enc = reinterpret_cast<EncodeTiledFn>(ptr);
    RMaps M;
    const int H = p.H;
    {
        const cuuint64_t dims[3] = {(cuuint64_t)H, (cuuint64_t)p.L0, (cuuint64_t)p.B};
        const cuuint64_t st[2] = {(cuuint64_t)H * 2, (cuuint64_t)p.L0 * H * 2};
        const cuuint32_t box[3] = {RBK, 1, RROWS};
        if (!enc_map(enc, &M.x, 3, t.x, dims, st, box, CU_TENSOR_MAP_SWIZZLE_128B, err)) return cudaErrorInvalidValue;
    }
    {
        const cuuint64_t dims[2] = {64, (cuuint64_t)hb_rows_total(p)};
        const cuuint64_t st[1] = {128};
        const cuuint32_t box[2] = {RBK, RROWS};
        if (!enc_map(enc, &M.h, 2, t.hb, dims, st, box, CU_TENSOR_MAP_SWIZZLE_128B, err)) return cudaErrorInvalidValue;
    }
    const CUtensorMapSwizzle wsw = BNUR == 16 ? CU_TENSOR_MAP_SWIZZLE_32B : CU_TENSOR_MAP_SWIZZLE_64B;
    {
        const cuuint64_t dims[4] = {(cuuint64_t)H, (cuuint64_t)H, 4, (cuuint64_t)p.D};
        const cuuint64_t st[3] = {(cuuint64_t)H * 2, (cuuint64_t)H * H * 2, (cuuint64_t)4 * H * H * 2};
        const cuuint32_t box[4] = {BNUR, RBK, 4, 1};
        if (!enc_map(enc, &M.W, 4, t.W, dims, st, box, wsw, err)) return cudaErrorInvalidValue;
        if (!enc_map(enc, &M.U, 4, t.U, dims, st, box, wsw, err)) return cudaErrorInvalidValue;
    }
    const size_t smem = resident_smem<BNUR>(H);
    e = cudaFuncSetAttribute(wavefront_resident_kernel<BNUR>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)smem);
    if (e != cudaSuccess) {
        if (err) *err = std::string("resident launch setup: ") + cudaGetErrorString(e);
        return e;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(p.D * (H / BNUR)));
    cfg.blockDim = dim3(RTHREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;  // every (layer, slab) CTA co-resident
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    e = cudaLaunchKernelEx(&cfg, wavefront_resident_kernel<BNUR>, p, t, M);
    if (e == cudaSuccess)
        set_last_launch("wavefront_resident_kernel<" + std::to_string(BNUR) + "> grid=" +
                        std::to_string(p.D * (H / BNUR)) + " cooperative=1");
    if (e != cudaSuccess && err) *err = std::string("resident launch: ") + cudaGetErrorString(e);
    return e;
}

}  // namespace

// Which resident slab width fits (0 = the weights cannot be resident): stacked only (every
// dilation 1), batch <= 128, one CTA per (layer, slab) on distinct SMs, slab + A ring <= 227 KB.
int resident_bnu(const Problem& p, int nsm) {
    if (p.kind != KIND_SEQ || p.cell != CELL_LSTM || p.B > RROWS || p.H % 64 != 0) return 0;
    for (int d = 0; d < p.D; ++d)
        if (p.dil[d] != 1) return 0;
    const size_t cap = 227 * 1024;
    if ((long long)p.D * (p.H / 16) <= nsm && resident_smem<16>(p.H) <= cap) return 16;
    if ((long long)p.D * (p.H / 32) <= nsm && resident_smem<32>(p.H) <= cap) return 32;
    return 0;
}

cudaError_t launch_wavefront_resident(const Problem& p, const Tensors& t, cudaStream_t s, int bnu,
                                      std::string* err) {
    return bnu == 16 ? launch_resident_t<16>(p, t, s, err) : launch_resident_t<32>(p, t, s, err);
}

}  // namespace ft
