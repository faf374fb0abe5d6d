// b2b_gemm.cu — NEXT-4: back-to-back GEMMs  D = (A @ B) @ C  (Table 6: K = 64,
// P = 64; 1.21x vs cuBLAS on A100, L393) as ONE tcgen05 kernel.  The intermediate S = A@B never
// leaves the SM: tcgen05.mma → TMEM (fp32) → tcgen05.ld → bf16 → swizzled SMEM → A operand of the
// second tcgen05.mma.  This is the "data reuse uncovered across operator boundaries" of the paper
// (§2) materialized on B200 on-chip memory.
//
// One CTA per 128-row block of A (M rows).  N is walked in chunks of 128:
//   GEMM1(j):  S_j[128 x 128]  = A_blk[128 x 64] · B[:, j*128 : j*128+128]     (TMEM buffer j%2)
//   convert :  S_j → bf16 → SMEM buffer j%2 (K-major, 128-byte swizzle)           (4 warps)
//   GEMM2(j):  D[128 x 64]   += S_j · C[j*128 : j*128+128, :]                    (TMEM)
// The MMA warp issues GEMM1(j+1) before GEMM2(j) so the tensor core works while S_j converts.
// Warps: 0 TMA producer (A once; B_j, C_j through a 3-stage ring), 1 MMA issuer, 2–5 converters /
// epilogue (one row per thread).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <string>

#include "ft_internal.h"
#include "ft_sm100.cuh"

namespace ft {
namespace {

using namespace sm100;

constexpr int BMr = 128;   // A rows per CTA (TMEM lanes)
constexpr int KD = 64;     // K of GEMM1
constexpr int PD = 64;     // P (N of GEMM2)
constexpr int NC = 128;    // N chunk (N of GEMM1, K of GEMM2)
constexpr int NSTAGE = 3;  // B/C chunk ring
constexpr int A_B = BMr * KD * 2;   // 16 KiB
constexpr int B_B = KD * NC * 2;    // 16 KiB: [2 n-atoms][64 k][64 n]
constexpr int C_B = NC * PD * 2;    // 16 KiB: [128 n rows][64 p]
constexpr int S_B = BMr * NC * 2;   // 32 KiB: [2 k-atoms][128 rows][64]
constexpr int B2_THREADS = 192;
constexpr int B2_SMEM = A_B + NSTAGE * (B_B + C_B) + 2 * S_B + 256 + 1024;
constexpr uint32_t IDESC1 = make_idesc_bf16_f32(BMr, NC, false, true);  // A K-major, B MN-major
constexpr uint32_t IDESC2 = make_idesc_bf16_f32(BMr, PD, false, true);  // S K-major, C MN-major
constexpr uint32_t TCOLS = 512;  // S0 [0,128) S1 [128,256) D [256,320)

struct B2Maps {
    CUtensorMap a, b, c;
};

__global__ void __launch_bounds__(B2_THREADS, 1)
b2b_gemm_kernel(const __grid_constant__ B2Maps M, int N, float* __restrict__ D) {
    extern __shared__ uint8_t smem_raw[];
    const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    uint8_t* smem = smem_raw + pad;
    uint8_t* sA = smem;
    uint8_t* sB = sA + A_B;
    uint8_t* sC = sB + NSTAGE * B_B;
    uint8_t* sS = sC + NSTAGE * C_B;
    uint64_t* bars = reinterpret_cast<uint64_t*>(sS + 2 * S_B);
    uint64_t* a_full = bars;
    uint64_t* bc_full = bars + 1;
    uint64_t* bc_empty = bc_full + NSTAGE;
    uint64_t* s_full = bc_empty + NSTAGE;   // [2] GEMM1 done → S in TMEM
    uint64_t* s_tfree = s_full + 2;         // [2] S TMEM buffer read by the converters
    uint64_t* ss_full = s_tfree + 2;        // [2] S written to SMEM
    uint64_t* ss_free = ss_full + 2;        // [2] GEMM2 done reading the SMEM buffer
    uint64_t* d_full = ss_free + 2;
    uint32_t* tslot = reinterpret_cast<uint32_t*>(d_full + 1);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int NJ = N / NC;
    if (threadIdx.x == 0) {
        mbar_init(a_full, 1);
        for (int s = 0; s < NSTAGE; ++s) {
            mbar_init(&bc_full[s], 1);
            mbar_init(&bc_empty[s], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&s_full[b], 1);
            mbar_init(&s_tfree[b], 4);
            mbar_init(&ss_full[b], 4);
            mbar_init(&ss_free[b], 1);
        }
        mbar_init(d_full, 1);
        fence_mbarrier_init();
    }
    if (warp == 1) tmem_alloc(tslot, TCOLS);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tslot;

    if (warp == 0) {
        if (lane == 0) {
            mbar_arrive_expect_tx(a_full, A_B);
            tma_load_2d_hint_addr<1>(smem_u32(sA), &M.a, smem_u32(a_full), 0, blockIdx.x * BMr,
                                     policy_evict_normal());
            const uint64_t keep = policy_evict_last();  // B and C are re-read by every CTA
            int st = 0;
            uint32_t ph = 0;
            for (int j = 0; j < NJ; ++j) {
                mbar_wait(&bc_empty[st], ph ^ 1);
                mbar_arrive_expect_tx(&bc_full[st], B_B + C_B);
                tma_load_3d_hint<1>(sB + st * B_B, &M.b, smem_u32(&bc_full[st]), 0, 0, 2 * j, keep);
                tma_load_2d_hint_addr<1>(smem_u32(sC + st * C_B), &M.c, smem_u32(&bc_full[st]), 0,
                                         j * NC, keep);
                if (++st == NSTAGE) {
                    st = 0;
                    ph ^= 1;
                }
            }
        }
    } else if (warp == 1) {
        {  // the whole warp (warp-uniform waits keep the MMA descriptors in uniform registers)
            mbar_wait_warp(a_full, 0);
            tc_fence_after();
            const uint64_t ad = make_sdesc(smem_u32(sA), 16, 1024);
            // B chunk: MN-major, two 64-n atoms 8 KiB apart (LBO), 8-k groups 1 KiB (SBO)
            const uint64_t bd0 = make_sdesc(smem_u32(sB), 8192, 1024);
            // C chunk: MN-major, one 64-p atom, 8-k groups 1 KiB apart
            const uint64_t cd0 = make_sdesc(smem_u32(sC), 8192, 1024);
            // S: K-major, two 64-k atoms 16 KiB apart, 8-row groups 1 KiB
            const uint64_t sd0 = make_sdesc(smem_u32(sS), 16, 1024);
            auto gemm1 = [&](int j) {
                const int st = j % NSTAGE;
                mbar_wait_warp(&bc_full[st], (uint32_t)((j / NSTAGE) & 1));
                mbar_wait_warp(&s_tfree[j & 1], (uint32_t)(((j >> 1) & 1) ^ 1));
                tc_fence_after();
                if (elect_one()) {
                    const uint64_t bd = bd0 + (uint64_t)((st * B_B) >> 4);
#pragma unroll
                    for (int kk = 0; kk < KD / 16; ++kk)
                        umma_f16(tmem + (uint32_t)((j & 1) * NC), ad + (uint64_t)((kk * 32) >> 4),
                                 bd + (uint64_t)((kk * 2048) >> 4), IDESC1, kk != 0);
                    umma_commit(&s_full[j & 1]);
                }
                __syncwarp();
            };
            gemm1(0);
            for (int j = 0; j < NJ; ++j) {
                if (j + 1 < NJ) gemm1(j + 1);
                mbar_wait_warp(&ss_full[j & 1], (uint32_t)((j >> 1) & 1));
                tc_fence_after();
                if (elect_one()) {
                    const int st = j % NSTAGE;
                    const uint64_t cd = cd0 + (uint64_t)((st * C_B) >> 4);
                    const uint64_t sd = sd0 + (uint64_t)(((j & 1) * S_B) >> 4);
#pragma unroll
                    for (int kk = 0; kk < NC / 16; ++kk)
                        umma_f16(tmem + 256u, sd + (uint64_t)((((kk >> 2) * 16384) + (kk & 3) * 32) >> 4),
                                 cd + (uint64_t)((kk * 2048) >> 4), IDESC2, (j | kk) != 0);
                    umma_commit(&ss_free[j & 1]);
                    umma_commit(&bc_empty[st]);
                }
                __syncwarp();
            }
            if (elect_one()) umma_commit(d_full);
            __syncwarp();
        }
    } else {
        const int q = warp & 3, row = q * 32 + lane;
        const uint32_t lane_off = (uint32_t)(q * 32) << 16;
        for (int j = 0; j < NJ; ++j) {
            const int b = j & 1;
            mbar_wait(&s_full[b], (uint32_t)((j >> 1) & 1));
            tc_fence_after();
            mbar_wait(&ss_free[b], (uint32_t)(((j >> 1) & 1) ^ 1));  // GEMM2(j-2) done with it
            uint8_t* srow = sS + b * S_B + row * 128;
#pragma unroll 1
            for (int half = 0; half < 2; ++half) {  // 64 columns = one 64-k atom of S
                float v[4][16];
                __syncwarp();
#pragma unroll
                for (int g = 0; g < 4; ++g)
                    tmem_ld_32x32b_x16(tmem + lane_off + (uint32_t)(b * NC + half * 64 + g * 16), v[g]);
                tmem_wait_ld();
                if (half == 1) {
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&s_tfree[b]);
                }
#pragma unroll
                for (int c = 0; c < 8; ++c) {  // 16-byte chunk c holds k = half*64 + c*8 ..
                    const float* f = &v[c >> 1][(c & 1) * 8];
                    __nv_bfloat162 p0 = __floats2bfloat162_rn(f[0], f[1]);
                    __nv_bfloat162 p1 = __floats2bfloat162_rn(f[2], f[3]);
                    __nv_bfloat162 p2 = __floats2bfloat162_rn(f[4], f[5]);
                    __nv_bfloat162 p3 = __floats2bfloat162_rn(f[6], f[7]);
                    uint4 w;
                    w.x = *reinterpret_cast<uint32_t*>(&p0);
                    w.y = *reinterpret_cast<uint32_t*>(&p1);
                    w.z = *reinterpret_cast<uint32_t*>(&p2);
                    w.w = *reinterpret_cast<uint32_t*>(&p3);
                    *reinterpret_cast<uint4*>(srow + half * 16384 + ((c ^ (row & 7)) * 16)) = w;
                }
            }
            // generic-proxy SMEM writes → visible to the tensor core's async-proxy reads
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            if (lane == 0) mbar_arrive(&ss_full[b]);
        }
        mbar_wait(d_full, 0);
        tc_fence_after();
        float dv[4][16];
        __syncwarp();
#pragma unroll
        for (int g = 0; g < 4; ++g) tmem_ld_32x32b_x16(tmem + lane_off + 256u + (uint32_t)(g * 16), dv[g]);
        tmem_wait_ld();
        float4* dst = reinterpret_cast<float4*>(D + ((long long)blockIdx.x * BMr + row) * PD);
#pragma unroll
        for (int g = 0; g < 4; ++g)
#pragma unroll
            for (int e = 0; e < 4; ++e)
                dst[g * 4 + e] = make_float4(dv[g][4 * e], dv[g][4 * e + 1], dv[g][4 * e + 2], dv[g][4 * e + 3]);
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc(tmem, TCOLS);
    }
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                          const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                          CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

bool enc2(EncFn enc, CUtensorMap* m, int rank, const void* base, const cuuint64_t* dims,
          const cuuint64_t* strides, const cuuint32_t* box, std::string* err) {
    const cuuint32_t es[3] = {1, 1, 1};
    if (enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, rank, const_cast<void*>(base), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
        if (err) *err = "cuTensorMapEncodeTiled (b2b) failed";
        return false;
    }
    return true;
}

}  // namespace

cudaError_t launch_b2b_gemm(int Mr, int N, const void* A, const void* B, const void* C, float* D,
                            cudaStream_t s, std::string* err) {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q = cudaDriverEntryPointSymbolNotFound;
    cudaError_t e = cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &ptr, 12000,
                                                     cudaEnableDefault, &q);
    if (e != cudaSuccess || !ptr) {
        if (err) *err = "cuTensorMapEncodeTiled not available";
        return cudaErrorNotSupported;
    }
    EncFn enc = reinterpret_cast<EncFn>(ptr);
    B2Maps M;
    {
        const cuuint64_t dims[2] = {(cuuint64_t)KD, (cuuint64_t)Mr};
        const cuuint64_t st[1] = {(cuuint64_t)KD * 2};
        const cuuint32_t box[2] = {64, (cuuint32_t)BMr};
        if (!enc2(enc, &M.a, 2, A, dims, st, box, err)) return cudaErrorInvalidValue;
    }
    {   // B [64][N] as (64 n_lo, 64 k, N/64 n_hi): one box = the two 64-n atoms of a chunk
        const cuuint64_t dims[3] = {64, (cuuint64_t)KD, (cuuint64_t)(N / 64)};
        const cuuint64_t st[2] = {(cuuint64_t)N * 2, 128};
        const cuuint32_t box[3] = {64, (cuuint32_t)KD, 2};
        if (!enc2(enc, &M.b, 3, B, dims, st, box, err)) return cudaErrorInvalidValue;
    }
    {
        const cuuint64_t dims[2] = {(cuuint64_t)PD, (cuuint64_t)N};
        const cuuint64_t st[1] = {(cuuint64_t)PD * 2};
        const cuuint32_t box[2] = {64, (cuuint32_t)NC};
        if (!enc2(enc, &M.c, 2, C, dims, st, box, err)) return cudaErrorInvalidValue;
    }
    e = cudaFuncSetAttribute(b2b_gemm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, B2_SMEM);
    if (e != cudaSuccess) {
        if (err) *err = std::string("b2b setup: ") + cudaGetErrorString(e);
        return e;
    }
    b2b_gemm_kernel<<<Mr / BMr, B2_THREADS, B2_SMEM, s>>>(M, N, D);
    e = cudaGetLastError();
    if (e != cudaSuccess && err) *err = std::string("b2b launch: ") + cudaGetErrorString(e);
    return e;
}

}  // namespace ft
