// layerwise.cu — NEXT-2: the layer-sequential schedule the paper argues against
// (the "DAG approach" that runs one layer after another, L67; the sub-linear depth hypothesis of
// Fig. 8), built the strongest way we know on B200 so the wavefront gets an honest
// comparison on the same box (cuDNN / Appleyard-style persistent RNN):
//
//   for d in 0..D-1:
//     1. hoisted input projection  Z_d = X_{d-1} @ W_d   — ONE large GEMM over all (batch, time)
//        rows (X_{-1} = x); a plain library GEMM (cuBLAS, loaded at run time), fp32 output;
//     2. the recurrence over t with U_d resident in shared memory: CTA (m, n) owns the 16-unit
//        slab U_d[:, gates, n*16 : n*16+16] for the whole sequence (TMA-loaded once) and batch
//        rows [m*128, m*128+128); per step it streams h_{t-1} (16 KiB K-chunks, TMA), runs
//        tcgen05.mma into TMEM, and the epilogue adds Z_d[t] + b_d, applies the LSTM update
//        (Listing 2; reading R1/R2) with c in registers, and releases a per-(t, m)
//        counter the other slabs of the same rows wait on.
//
// Same results as ft_stacked_lstm_fwd up to fp32 summation order (the input and recurrent halves
// are summed in a different order); the layer-sequential order is legal because every
// dependence distance of the nest is non-negative (Table 4).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstdlib>
#include <string>

#include "ft_internal.h"
#include "ft_sm100.cuh"

namespace ft {
namespace {

using namespace sm100;

constexpr int LROWS = 128;     // batch rows per CTA (one UMMA M)
constexpr int LBK = 64;        // K chunk
constexpr int LBNU = 16;       // units per slab → UMMA N = 64
constexpr int LN = 4 * LBNU;
constexpr int LTHREADS = 192;  // warp 0 TMA, warp 1 MMA, warps 2–5 epilogue
constexpr int LSTAGES_MAX = 12;  // A ring depth: as deep as the U slab leaves room for
constexpr int LSW = LBNU * 2;                       // bytes per weight smem row (32-byte swizzle)
constexpr int LGATE_BYTES = LBNU * LBK * 2;         // 2 KiB: one gate atom column of a K chunk
constexpr int LWCHUNK = 4 * LGATE_BYTES;            // 8 KiB: one K chunk of the slab
constexpr int LA_BYTES = LROWS * LBK * 2;           // 16 KiB
constexpr int LTMEM_COLS = 2 * LN;                  // double-buffered accumulator
constexpr uint32_t LIDESC = make_idesc_bf16_f32(LROWS, LN, false, true);

struct LayerArgs {
    int B, T, H, D, d, MB, NTR;
    int stages;            // A ring depth (shared memory left after the U slab)
    int debug;             // development builds only (FT_DEV_EXPERIMENTS, env FT_DEBUG): 8 = skip
                           // the A loads (wrong results); always 0 in libft.so
    int a_rows;            // rows per A box: min(128, batch rounded up to 8) — no padded-row loads
    const float* Z;        // [B][T][4H] fp32 = X_{d-1} @ W_d (gate-major columns)
    const float* b;        // [4][H] bias of layer d
    __nv_bfloat16* out;    // [B][T][H] layer output (y for the top layer)
    __nv_bfloat16* hb;     // blocked h of this layer [T][H/64][MB*128][64] (A operand source)
    __nv_bfloat16* h_all;  // optional [B][D][T][H]
    float* c_all;          // optional [B][D][T][H]
    __nv_bfloat16* h_n;    // [B][D][H]
    float* c_n;            // [B][D][H]
    int* flags;            // [T][MB] for this layer
};

#ifdef FT_TRACE
// development-only step timeline of CTA 0 (libft_trace.so): per (layer, step) six %globaltimer
// stamps — 0 producer saw h_{t-1} ready, 1 MMA saw the first A chunk, 2 last MMA issued,
// 3 epilogue saw the accumulator, 4 h stored (before the release), 5 released
constexpr int LW_EV_MAX = 64 * 1024;
__device__ unsigned long long g_lw_events[LW_EV_MAX * 6];
#define LW_EV(cond, d, t, k)                                                                  \
    do {                                                                                      \
        if ((cond) && blockIdx.x == 0 && (long long)(d) * A.T + (t) < LW_EV_MAX)             \
            g_lw_events[((long long)(d) * A.T + (t)) * 6 + (k)] = globaltimer_ns();           \
    } while (0)
#else
#define LW_EV(cond, d, t, k) ((void)0)
#endif

struct LayerMaps {
    CUtensorMap U, hb;
};

__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
    __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
    return *reinterpret_cast<uint32_t*>(&v);
}

__global__ void __launch_bounds__(LTHREADS, 1)
layer_recurrent_kernel(const __grid_constant__ LayerArgs A, const __grid_constant__ LayerMaps M) {
    extern __shared__ uint8_t smem_raw[];
    const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    uint8_t* smem = smem_raw + pad;
    const int KCH = A.H / LBK;
    const int Bp = A.MB * LROWS;
    uint8_t* sU = smem;                       // KCH resident chunks of the U slab
    uint8_t* sA = smem + KCH * LWCHUNK;       // A ring
    const int S = A.stages;
    uint64_t* bars = reinterpret_cast<uint64_t*>(sA + S * LA_BYTES);
    uint64_t* full = bars;
    uint64_t* empty = bars + S;
    uint64_t* tfull = bars + 2 * S;
    uint64_t* tempty = tfull + 2;
    uint64_t* wbar = tempty + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(wbar + 1);

    const int m = blockIdx.x / A.NTR, n = blockIdx.x % A.NTR;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
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
    if (warp == 1) tmem_alloc(tmem_slot, LTMEM_COLS);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {
            const uint64_t pol_keep = policy_evict_last();
            const uint64_t pol_act = policy_evict_normal();
            mbar_arrive_expect_tx(wbar, KCH * LWCHUNK);
            for (int c = 0; c < KCH; ++c)
                tma_load_4d_hint_addr<1>(smem_u32(sU + c * LWCHUNK), &M.U, smem_u32(wbar), n * LBNU,
                                         c * LBK, 0, A.d, pol_keep);
            int stage = 0;
            uint32_t phase = 0;
            for (int t = 1; t < A.T; ++t) {
                wait_flag_geq(A.flags + (long long)(t - 1) * A.MB + m, A.NTR);
                LW_EV(true, A.d, t, 0);
                fence_proxy_async_global();
                for (int kc = 0; kc < KCH; ++kc) {
                    mbar_wait(&empty[stage], phase ^ 1);
                    if (FT_DEV_BIT(A.debug, 8)) {
                        mbar_arrive(&full[stage]);
                        if (++stage == S) {
                            stage = 0;
                            phase ^= 1;
                        }
                        continue;
                    }
                    mbar_arrive_expect_tx(&full[stage], A.a_rows * 128);
                    tma_load_2d_hint_addr<1>(smem_u32(sA + stage * LA_BYTES), &M.hb,
                                             smem_u32(&full[stage]), 0,
                                             (int)(((long long)(t - 1) * KCH + kc) * Bp + m * LROWS),
                                             pol_act);
                    if (++stage == S) {
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
            // U slab: MN-major, 16-unit (32-byte swizzle) atoms, gates LGATE_BYTES apart (LBO),
            // 8-k-row groups 8*LSW apart (SBO); a K step of 16 rows is 16*LSW bytes.
            const uint64_t bdesc0 = make_sdesc(smem_u32(sU), LGATE_BYTES, 8 * LSW, 6u);
            int stage = 0, acc = 0;
            uint32_t phase = 0, acc_phase = 0;
            for (int t = 1; t < A.T; ++t) {
                mbar_wait_warp(&tempty[acc], acc_phase ^ 1);
                tc_fence_after();
                const uint32_t d_tmem = tmem_base + (uint32_t)(acc * LN);
                for (int kc = 0; kc < KCH; ++kc) {
                    mbar_wait_warp(&full[stage], phase);
                    LW_EV(kc == 0, A.d, t, 1);
                    tc_fence_after();
                    if (elect_one()) {
                        const uint64_t ad = adesc0 + (uint64_t)((stage * LA_BYTES) >> 4);
                        const uint64_t bd = bdesc0 + (uint64_t)((kc * LWCHUNK) >> 4);
#pragma unroll
                        for (int kk = 0; kk < LBK / 16; ++kk)
                            umma_f16(d_tmem, ad + (uint64_t)((kk * 32) >> 4),
                                     bd + (uint64_t)((kk * 16 * LSW) >> 4), LIDESC, (kc | kk) != 0);
                        umma_commit(&empty[stage]);
                    }
                    __syncwarp();
                    if (++stage == S) {
                        stage = 0;
                        phase ^= 1;
                    }
                }
                if (elect_one()) umma_commit(&tfull[acc]);
                __syncwarp();
                LW_EV(true, A.d, t, 2);
                acc ^= 1;
                if (acc == 0) acc_phase ^= 1;
            }
        }
    } else {
        // ---- epilogue: one batch row per thread, the slab's 16 units x 4 gates --------------
        const int q = warp & 3, row = m * LROWS + q * 32 + lane;
        const bool valid = row < A.B;
        const int n0 = n * LBNU;
        const int H = A.H;
        float creg[LBNU];
#pragma unroll
        for (int u = 0; u < LBNU; ++u) creg[u] = 0.f;
        int acc = 0;
        uint32_t acc_phase = 0;
        for (int t = 0; t < A.T; ++t) {
            // the hoisted projection of this step does not depend on the recurrence: load it
            // while the MMAs for h_{t-1} @ U run
            float z[4][LBNU];
            if (valid) {
                const float4* zr = reinterpret_cast<const float4*>(A.Z + ((long long)row * A.T + t) * 4 * H + n0);
#pragma unroll
                for (int g = 0; g < 4; ++g)
#pragma unroll
                    for (int w = 0; w < LBNU / 4; ++w) {
                        const float4 v = __ldcs(zr + (g * H) / 4 + w);
                        z[g][4 * w + 0] = v.x;
                        z[g][4 * w + 1] = v.y;
                        z[g][4 * w + 2] = v.z;
                        z[g][4 * w + 3] = v.w;
                    }
            } else {
#pragma unroll
                for (int g = 0; g < 4; ++g)
#pragma unroll
                    for (int u = 0; u < LBNU; ++u) z[g][u] = 0.f;
            }
            if (t > 0) {
                mbar_wait(&tfull[acc], acc_phase);
                LW_EV(threadIdx.x == 64, A.d, t, 3);
                tc_fence_after();
                const uint32_t tbase = tmem_base + (uint32_t)(acc * LN) + ((uint32_t)(q * 32) << 16);
                float r[4][16];
                tmem_ld_32x32b_x16(tbase + 0 * LBNU, r[0]);
                tmem_ld_32x32b_x16(tbase + 1 * LBNU, r[1]);
                tmem_ld_32x32b_x16(tbase + 2 * LBNU, r[2]);
                tmem_ld_32x32b_x16(tbase + 3 * LBNU, r[3]);
                tmem_wait_ld();
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&tempty[acc]);
#pragma unroll
                for (int g = 0; g < 4; ++g)
#pragma unroll
                    for (int u = 0; u < LBNU; ++u) z[g][u] += r[g][u];
                acc ^= 1;
                if (acc == 0) acc_phase ^= 1;
            }
            float hv[LBNU];
            const float* bias = A.b + n0;
#pragma unroll
            for (int u = 0; u < LBNU; ++u) {
                const float ig = sigmoid_approx(z[0][u] + __ldg(bias + 0 * H + u));
                const float fg = sigmoid_approx(z[1][u] + __ldg(bias + 1 * H + u));
                const float og = sigmoid_approx(z[2][u] + __ldg(bias + 2 * H + u));
                const float gh = tanh_approx(z[3][u] + __ldg(bias + 3 * H + u));
                creg[u] = fmaf(fg, creg[u], ig * gh);
                hv[u] = og * tanh_approx(creg[u]);
            }
            uint32_t hp[LBNU / 2];
#pragma unroll
            for (int v = 0; v < LBNU / 2; ++v) hp[v] = pack2(hv[2 * v], hv[2 * v + 1]);
            if (valid && t + 1 < A.T) {
                uint4* dst = reinterpret_cast<uint4*>(
                    A.hb + (((long long)t * (H / 64) + n0 / 64) * (A.MB * LROWS) + row) * 64 + (n0 % 64));
                __stcg(dst + 0, make_uint4(hp[0], hp[1], hp[2], hp[3]));
                __stcg(dst + 1, make_uint4(hp[4], hp[5], hp[6], hp[7]));
            }
            named_bar_sync(1, 128);
            if (threadIdx.x == 64 && t + 1 < A.T) {
                LW_EV(true, A.d, t, 4);
                fence_acq_rel_gpu();
                red_release_gpu_add(A.flags + (long long)t * A.MB + m, 1);
                LW_EV(true, A.d, t, 5);
            }
            if (valid) {  // outputs the recurrence does not read
                uint4* dy = reinterpret_cast<uint4*>(A.out + ((long long)row * A.T + t) * H + n0);
                dy[0] = make_uint4(hp[0], hp[1], hp[2], hp[3]);
                dy[1] = make_uint4(hp[4], hp[5], hp[6], hp[7]);
                const long long hi = (((long long)row * A.D + A.d) * A.T + t) * H + n0;
                if (A.h_all) {
                    uint4* dh = reinterpret_cast<uint4*>(A.h_all + hi);
                    dh[0] = make_uint4(hp[0], hp[1], hp[2], hp[3]);
                    dh[1] = make_uint4(hp[4], hp[5], hp[6], hp[7]);
                }
                if (A.c_all) {
                    float4* dc = reinterpret_cast<float4*>(A.c_all + hi);
#pragma unroll
                    for (int w = 0; w < LBNU / 4; ++w)
                        dc[w] = make_float4(creg[4 * w], creg[4 * w + 1], creg[4 * w + 2], creg[4 * w + 3]);
                }
                if (t == A.T - 1) {
                    const long long ni = ((long long)row * A.D + A.d) * H + n0;
                    uint4* dn = reinterpret_cast<uint4*>(A.h_n + ni);
                    dn[0] = make_uint4(hp[0], hp[1], hp[2], hp[3]);
                    dn[1] = make_uint4(hp[4], hp[5], hp[6], hp[7]);
                    float4* dc = reinterpret_cast<float4*>(A.c_n + ni);
#pragma unroll
                    for (int w = 0; w < LBNU / 4; ++w)
                        dc[w] = make_float4(creg[4 * w], creg[4 * w + 1], creg[4 * w + 2], creg[4 * w + 3]);
                }
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc(tmem_base, LTMEM_COLS);
    }
}

// ---------------------------------------------------------------------------------------------
// host side

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// cuBLAS is loaded at run time (only this comparison schedule uses it), so libft.so itself has
// no link-time dependency on it.  Types mirror cublas_api.h (cublasStatus_t / enums are ints).
typedef int (*CublasCreateFn)(void**);
typedef int (*CublasSetStreamFn)(void*, cudaStream_t);
typedef int (*CublasGemmSBEx)(void*, int, int, int, int, int, const void*, const void*, int, int,
                              long long, const void*, int, int, long long, const void*, void*, int,
                              int, long long, int, int, int);
constexpr int CUBLAS_OP_N_ = 0;
constexpr int CUDA_R_32F_ = 0, CUDA_R_16BF_ = 14;
constexpr int CUBLAS_COMPUTE_32F_ = 68, CUBLAS_GEMM_DEFAULT_ = -1;

struct Cublas {
    void* lib = nullptr;
    CublasCreateFn create = nullptr;
    CublasSetStreamFn set_stream = nullptr;
    CublasGemmSBEx gemm = nullptr;
    void* handle[16] = {};
};

Cublas* cublas(std::string* err) {
    static Cublas c;
    if (!c.lib) {
        const char* names[] = {"libcublas.so.12", "/usr/local/cuda/lib64/libcublas.so.12"};
        for (const char* nm : names)
            if ((c.lib = dlopen(nm, RTLD_NOW | RTLD_GLOBAL))) break;
        if (!c.lib) {
            if (err) *err = "libcublas.so.12 not found (layer-sequential schedule needs cuBLAS)";
            return nullptr;
        }
        c.create = (CublasCreateFn)dlsym(c.lib, "cublasCreate_v2");
        c.set_stream = (CublasSetStreamFn)dlsym(c.lib, "cublasSetStream_v2");
        c.gemm = (CublasGemmSBEx)dlsym(c.lib, "cublasGemmStridedBatchedEx");
        if (!c.create || !c.set_stream || !c.gemm) {
            if (err) *err = "cuBLAS symbols missing";
            c.lib = nullptr;
            return nullptr;
        }
    }
    return &c;
}

size_t layer_smem(int H, int stages) {
    return (size_t)(H / LBK) * LWCHUNK + (size_t)stages * LA_BYTES + 16 * (2 * stages + 5) + 1024;
}
int layer_stages(int H) {
    int s = LSTAGES_MAX;
    while (s > 2 && layer_smem(H, s) > 227 * 1024) --s;
    return s;
}

}  // namespace

#ifdef FT_TRACE
extern "C" __attribute__((visibility("default"))) int ft_debug_lw_events(unsigned long long* host, int n) {
    if (n > LW_EV_MAX) n = LW_EV_MAX;
    cudaDeviceSynchronize();
    if (cudaMemcpyFromSymbol(host, g_lw_events, (size_t)n * 6 * sizeof(unsigned long long)) != cudaSuccess)
        return -1;
    return n;
}
#endif

// Whether the layer-sequential schedule supports the shape on this device (0 = yes).
int layerwise_supported(int B, int H, int nsm, std::string* why) {
    const int MB = (B + LROWS - 1) / LROWS;
    if (H % 64 != 0) {
        *why = "hidden % 64 != 0";
        return 1;
    }
    if ((long long)MB * (H / LBNU) > nsm) {
        *why = "ceil(batch/128) * hidden/16 CTAs exceed the SM count (the recurrence is one co-resident grid)";
        return 1;
    }
    if (layer_smem(H, 2) > 227 * 1024) {
        *why = "the U slab (hidden x 64 bf16) does not fit in shared memory";
        return 1;
    }
    return 0;
}

size_t layerwise_ws_bytes(int B, int T, int H) {
    const size_t MB = (B + LROWS - 1) / LROWS;
    auto r = [](size_t v) { return (v + 255) / 256 * 256; };
    return r((size_t)B * T * 4 * H * 4)          // Z fp32
           + 2 * r((size_t)B * T * H * 2)        // ping-pong layer outputs
           + r((size_t)T * H * MB * LROWS * 2)   // blocked h of the current layer
           + r((size_t)T * MB * 4) * 64;         // counters (up to FT_MAX_DEPTH layers)
}

cudaError_t launch_layerwise(int B, int T, int H, int D, const void* x, const void* W, const void* U,
                             const float* b, void* y, void* h_n, float* c_n, void* h_all,
                             float* c_all, void* ws, cudaStream_t s, std::string* err) {
    Cublas* cb = cublas(err);
    if (!cb) return cudaErrorNotSupported;
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 16) return cudaErrorInvalidDevice;
    if (!cb->handle[dev] && cb->create(&cb->handle[dev]) != 0) {
        if (err) *err = "cublasCreate failed";
        return cudaErrorUnknown;
    }
    void* hdl = cb->handle[dev];
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q = cudaDriverEntryPointSymbolNotFound;
    cudaError_t e = cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &ptr, 12000, cudaEnableDefault, &q);
    if (e != cudaSuccess || !ptr) {
        if (err) *err = "cuTensorMapEncodeTiled not available";
        return cudaErrorNotSupported;
    }
    EncodeTiledFn enc = reinterpret_cast<EncodeTiledFn>(ptr);

    const int MB = (B + LROWS - 1) / LROWS, NTR = H / LBNU;
    auto r = [](size_t v) { return (v + 255) / 256 * 256; };
    uint8_t* p = static_cast<uint8_t*>(ws);
    float* Z = reinterpret_cast<float*>(p);
    p += r((size_t)B * T * 4 * H * 4);
    __nv_bfloat16* ping[2];
    ping[0] = reinterpret_cast<__nv_bfloat16*>(p);
    p += r((size_t)B * T * H * 2);
    ping[1] = reinterpret_cast<__nv_bfloat16*>(p);
    p += r((size_t)B * T * H * 2);
    __nv_bfloat16* hb = reinterpret_cast<__nv_bfloat16*>(p);
    p += r((size_t)T * H * MB * LROWS * 2);
    int* flags = reinterpret_cast<int*>(p);
    const size_t flag_stride = r((size_t)T * MB * 4);

    const int stages = layer_stages(H);
    const int a_rows = B >= LROWS ? LROWS : (B + 7) / 8 * 8;
    LayerMaps M;
    const cuuint32_t es[4] = {1, 1, 1, 1};
    {
        const cuuint64_t dims[4] = {(cuuint64_t)H, (cuuint64_t)H, 4, (cuuint64_t)D};
        const cuuint64_t st[3] = {(cuuint64_t)H * 2, (cuuint64_t)H * H * 2, (cuuint64_t)4 * H * H * 2};
        const cuuint32_t box[4] = {LBNU, LBK, 4, 1};
        if (enc(&M.U, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(U), dims, st, box, es,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
            if (err) *err = "cuTensorMapEncodeTiled (layerwise U) failed";
            return cudaErrorInvalidValue;
        }
    }
    {
        const cuuint64_t dims[2] = {64, (cuuint64_t)T * (H / 64) * MB * LROWS};
        const cuuint64_t st[1] = {128};
        const cuuint32_t box[2] = {LBK, (cuuint32_t)a_rows};
        if (enc(&M.hb, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, hb, dims, st, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
            if (err) *err = "cuTensorMapEncodeTiled (layerwise hb) failed";
            return cudaErrorInvalidValue;
        }
    }
    const size_t smem = layer_smem(H, stages);
    e = cudaFuncSetAttribute(layer_recurrent_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) e = cudaMemsetAsync(flags, 0, flag_stride * D, s);
    if (e != cudaSuccess) {
        if (err) *err = std::string("layerwise setup: ") + cudaGetErrorString(e);
        return e;
    }
    if (cb->set_stream(hdl, s) != 0) {
        if (err) *err = "cublasSetStream failed";
        return cudaErrorUnknown;
    }
    const float one = 1.f, zero = 0.f;
    const __nv_bfloat16* X = static_cast<const __nv_bfloat16*>(x);
    for (int d = 0; d < D; ++d) {
        // 1. Z[m][g*H + n] = sum_k X[m][k] W[d][g][k][n], m over all B*T (batch, time) rows.
        //    Column-major view: Z_g^T (H x BT, ld 4H) = W_g^T (H x H, ld H) * X^T (H x BT, ld H).
        const __nv_bfloat16* Wd = static_cast<const __nv_bfloat16*>(W) + (size_t)d * 4 * H * H;
        int st = cb->gemm(hdl, CUBLAS_OP_N_, CUBLAS_OP_N_, H, B * T, H, &one, Wd, CUDA_R_16BF_, H,
                          (long long)H * H, X, CUDA_R_16BF_, H, 0, &zero, Z, CUDA_R_32F_, 4 * H, H, 4,
                          CUBLAS_COMPUTE_32F_, CUBLAS_GEMM_DEFAULT_);
        if (st != 0) {
            if (err) *err = "cublasGemmStridedBatchedEx failed: " + std::to_string(st);
            return cudaErrorUnknown;
        }
        // 2. the recurrence of layer d
        LayerArgs a;
        a.B = B;
        a.T = T;
        a.H = H;
        a.D = D;
        a.d = d;
        a.MB = MB;
        a.NTR = NTR;
        a.stages = stages;
#ifdef FT_DEV_EXPERIMENTS  // development builds only (tools/variant_build.sh); never in libft.so
        a.debug = getenv("FT_DEBUG") ? atoi(getenv("FT_DEBUG")) : 0;
#else
        a.debug = 0;
#endif
        a.a_rows = a_rows;
        a.Z = Z;
        a.b = b + (size_t)d * 4 * H;
        a.out = d == D - 1 ? static_cast<__nv_bfloat16*>(y) : ping[d & 1];
        a.hb = hb;
        a.h_all = static_cast<__nv_bfloat16*>(h_all);
        a.c_all = c_all;
        a.h_n = static_cast<__nv_bfloat16*>(h_n);
        a.c_n = c_n;
        a.flags = reinterpret_cast<int*>(reinterpret_cast<uint8_t*>(flags) + flag_stride * d);
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3((unsigned)(MB * NTR));
        cfg.blockDim = dim3(LTHREADS);
        cfg.dynamicSmemBytes = smem;
        cfg.stream = s;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeCooperative;  // the slabs of one row block spin on each other
        attr[0].val.cooperative = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        e = cudaLaunchKernelEx(&cfg, layer_recurrent_kernel, a, M);
        if (e != cudaSuccess) {
            if (err) *err = std::string("layerwise launch: ") + cudaGetErrorString(e);
            return e;
        }
        set_last_launch("layerwise: per layer cuBLAS input GEMM + layer_recurrent_kernel grid=" +
                        std::to_string(MB * NTR) + " cooperative=1 (x" + std::to_string(D) + " layers)");
        X = a.out;
    }
    return cudaSuccess;
}

}  // namespace ft
