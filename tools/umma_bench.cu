// umma_bench.cu — development microbenchmark: tcgen05.mma kind::f16 issue-to-completion rate per
// SM for M = 128 and different N / B-operand layouts (operands are zeros in shared memory; only
// timing matters).  Not part of the library.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_sosp_liuqc0hs0y24_b200/csrc \
//        -o build/umma_bench tools/umma_bench.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdint>

#include "ft_sm100.cuh"

using namespace ft::sm100;

struct Cfg {
    const char* name;
    int N;
    bool b_mn;
    uint32_t layout, lbo, sbo;
    int kstep_bytes;  // B descriptor advance per K16 step
};

// mode 0: alternate two accumulators every 4 MMAs; 1: one accumulator; 2: one accumulator +
// tcgen05.commit every 4 MMAs (ring of 6 barriers, never waited); 3: as 2, and the issuer waits for
// the commit of chunk i-6 before chunk i (an SMEM ring's back-pressure)
// mode 5: mode 4 without tcgen05.fence::after_thread_sync; mode 6: mode 4 without the wait
// mode 4: the layer kernel's MMA loop shape: per 64-deep chunk wait a (pre-completed) ring
// barrier, 4 unrolled MMAs into one accumulator, commit to the ring
__device__ __forceinline__ void wait_test_spin(uint64_t* bar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.test_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
}
__device__ __forceinline__ void wait_relaxed(uint64_t* bar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.relaxed.cta.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
}
__device__ __forceinline__ void wait_try_hint(uint64_t* bar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2, %3;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(smem_u32(bar)), "r"(parity), "r"(20)
            : "memory");
}

template <int mode>
__global__ void __launch_bounds__(128, 1) umma_loop(Cfg c, int iters, unsigned long long* out) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    uint8_t* smem = smem_raw + pad;
    uint8_t* sA = smem;              // 64 KiB
    uint8_t* sB = smem + 65536;      // 64 KiB
    uint64_t* bar = reinterpret_cast<uint64_t*>(smem + 131072);
    uint64_t* ring = bar + 1;
    uint32_t* slot = reinterpret_cast<uint32_t*>(bar + 32);
    for (int i = threadIdx.x; i < 131072 / 16; i += blockDim.x)
        reinterpret_cast<uint4*>(smem)[i] = make_uint4(0, 0, 0, 0);
    if (threadIdx.x == 0) {
        mbar_init(bar, 1);
        for (int i = 0; i < 24; ++i) mbar_init(&ring[i], 1);
        fence_mbarrier_init();
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (threadIdx.x < 32) tmem_alloc(slot, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *slot;
    if constexpr (mode == 23) {
        // the whole warp runs the loop; warp-uniform waits (vote); one elected lane issues
        if (threadIdx.x < 32) {
            if (threadIdx.x == 0) mbar_arrive(&ring[23]);
            __syncwarp();
            const uint32_t idesc = make_idesc_bf16_f32(128, c.N, false, c.b_mn);
            const uint64_t a0 = make_sdesc(smem_u32(sA), 16, 1024, 2);
            const uint64_t b0 = make_sdesc(smem_u32(sB), c.lbo, c.sbo, c.layout);
            const long long t0 = clock64();
            for (int chunk = 0; chunk < iters / 4; ++chunk) {
                while (!__all_sync(0xffffffffu, mbar_try_wait(&ring[23], 0))) {
                }
                tc_fence_after();
                uint32_t is_leader;
                asm volatile("{\n\t.reg .pred p;\n\telect.sync _|p, 0xffffffff;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                             : "=r"(is_leader));
                if (is_leader) {
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk)
                        umma_f16(tmem, a0 + (uint64_t)((kk * 32) >> 4), b0 + (uint64_t)((kk * c.kstep_bytes) >> 4),
                                 idesc, (chunk | kk) != 0);
                    umma_commit(&ring[chunk % 6]);
                }
                __syncwarp();
            }
            if (threadIdx.x == 0) {
                umma_commit(bar);
                mbar_wait(bar, 0);
                out[blockIdx.x] = (unsigned long long)(clock64() - t0);
            }
        }
    } else if constexpr (mode == 21) {
        if (threadIdx.x < 32) {
            if (threadIdx.x == 0) mbar_arrive(&ring[23]);
            __syncwarp();
            const uint32_t idesc = make_idesc_bf16_f32(128, c.N, false, c.b_mn);
            const uint64_t a0 = make_sdesc(smem_u32(sA), 16, 1024, 2);
            const uint64_t b0 = make_sdesc(smem_u32(sB), c.lbo, c.sbo, c.layout);
            const long long t0 = clock64();
            for (int chunk = 0; chunk < iters / 4; ++chunk) {
                if (threadIdx.x == 1) mbar_wait(&ring[23], 0);
                __syncwarp();
                if (threadIdx.x == 0) {
                    tc_fence_after();
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk)
                        umma_f16(tmem, a0 + (uint64_t)((kk * 32) >> 4), b0 + (uint64_t)((kk * c.kstep_bytes) >> 4),
                                 idesc, (chunk | kk) != 0);
                    umma_commit(&ring[chunk % 6]);
                }
            }
            if (threadIdx.x == 0) {
                umma_commit(bar);
                mbar_wait(bar, 0);
                out[blockIdx.x] = (unsigned long long)(clock64() - t0);
            }
        }
    } else if (threadIdx.x == 0) {
        const uint32_t idesc = make_idesc_bf16_f32(128, c.N, false, c.b_mn);
        const uint64_t a0 = make_sdesc(smem_u32(sA), 16, 1024, 2);
        const uint64_t b0 = make_sdesc(smem_u32(sB), c.lbo, c.sbo, c.layout);
        const long long t0 = clock64();
        if constexpr (mode >= 7 && mode < 14) {
            // latency: batches of nb = 1 << (mode - 7) MMAs, each followed by commit + wait
            const int nb = 1 << (mode - 7);
            uint32_t phase = 0;
            for (int r = 0; r < iters / nb; ++r) {
                for (int k = 0; k < nb; ++k)
                    umma_f16(tmem, a0 + (uint64_t)(((k & 3) * 32) >> 4),
                             b0 + (uint64_t)(((k & 3) * c.kstep_bytes) >> 4), idesc, k != 0);
                umma_commit(&ring[0]);
                mbar_wait(&ring[0], phase);
                phase ^= 1;
            }
        } else if constexpr (mode >= 4) {
            // ring depth: modes 16/17/18 = 12/3/24 barriers, else 6
            constexpr int DEPTH = mode == 16 ? 12 : mode == 17 ? 3 : mode == 18 ? 24 : 6;
            // mode 19: wait on an already-complete plain barrier each chunk; 20: relaxed wait on the ring
            if ((mode == 19 || mode == 22) && threadIdx.x == 0) mbar_arrive(&ring[23]);
            int stage = 0;
            uint32_t phase = 0;
            for (int chunk = 0; chunk < iters / 4; ++chunk) {
                if (mode == 14 && chunk >= DEPTH) wait_test_spin(&ring[stage], phase ^ 1);
                if (mode == 15 && chunk >= DEPTH) wait_try_hint(&ring[stage], phase ^ 1);
                if (mode == 19 || (mode == 22 && (chunk & 1) == 0)) mbar_wait(&ring[23], 0);
                if (mode == 20 && chunk >= DEPTH) wait_relaxed(&ring[stage], phase ^ 1);
                if ((mode < 14 || (mode >= 16 && mode < 19)) && mode != 6 && chunk >= DEPTH) mbar_wait(&ring[stage], phase ^ 1);
                if (mode != 5) tc_fence_after();
#pragma unroll
                for (int kk = 0; kk < 4; ++kk)
                    umma_f16(tmem, a0 + (uint64_t)((kk * 32) >> 4), b0 + (uint64_t)((kk * c.kstep_bytes) >> 4),
                             idesc, (chunk | kk) != 0);
                umma_commit(&ring[stage]);
                if (++stage == DEPTH) {
                    stage = 0;
                    phase ^= 1;
                }
            }
        }
        uint32_t ph[6] = {0, 0, 0, 0, 0, 0};
        for (int it = 0; it < (mode >= 4 ? 0 : iters); ++it) {  // modes 0-3
            const int kk = it & 3;
            const int chunk = it >> 2;
            if (mode == 3 && kk == 0 && chunk >= 6) {
                mbar_wait(&ring[chunk % 6], ph[chunk % 6]);
                ph[chunk % 6] ^= 1;
            }
            const uint32_t d = tmem + (mode == 0 ? (uint32_t)(chunk & 1) * 256 : 0u);
            umma_f16(d, a0 + (uint64_t)((kk * 32) >> 4), b0 + (uint64_t)((kk * c.kstep_bytes) >> 4), idesc,
                     mode == 0 ? kk != 0 : it != 0);
            if (mode >= 2 && kk == 3) umma_commit(&ring[chunk % 6]);
        }
        umma_commit(bar);
        mbar_wait(bar, 0);
        const long long t1 = clock64();
        out[blockIdx.x] = (unsigned long long)(t1 - t0);
    }
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x < 32) {
        tc_fence_after();
        tmem_dealloc(tmem, 512);
    }
}

int main() {
    const Cfg cfgs[] = {
        {"N256 B MN-major SW128 (hot path)", 256, true, 2, 8192, 1024, 16 * 128},
        {"N128 B MN-major SW64  (32-unit tiles)", 128, true, 4, 4096, 512, 16 * 64},
        {"N64  B MN-major SW32  (16-unit slabs)", 64, true, 6, 2048, 256, 16 * 32},
        {"N64  B MN-major SW128 (one 64-col atom)", 64, true, 2, 8192, 1024, 16 * 128},
        {"N256 B K-major SW128", 256, false, 2, 16, 1024, 32},
        {"N128 B K-major SW128", 128, false, 2, 16, 1024, 32},
        {"N64  B K-major SW128", 64, false, 2, 16, 1024, 32},
        {"N32  B K-major SW128", 32, false, 2, 16, 1024, 32},
    };
    unsigned long long* d_out;
    cudaMalloc(&d_out, 1024 * sizeof(unsigned long long));
    const int smem = 131072 + 2048;
    cudaFuncSetAttribute(umma_loop<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<5>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<6>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<7>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<9>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<11>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<13>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<14>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<15>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<17>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<18>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<19>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<20>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<21>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<22>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(umma_loop<23>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    void (*kern[24])(Cfg, int, unsigned long long*) = {umma_loop<0>, umma_loop<1>, umma_loop<2>, umma_loop<3>,
                                                      umma_loop<4>, umma_loop<5>, umma_loop<6>, umma_loop<7>,
                                                      nullptr, umma_loop<9>, nullptr, umma_loop<11>, nullptr,
                                                      umma_loop<13>, umma_loop<14>, umma_loop<15>,
                                                      umma_loop<16>, umma_loop<17>, umma_loop<18>,
                                                      umma_loop<19>, umma_loop<20>, umma_loop<21>,
                                                      umma_loop<22>, umma_loop<23>};
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const int iters = 8192;
    for (const Cfg& c : cfgs) {
        for (int mode = 4; mode < 24; ++mode) {
            if (mode == 5 || (mode >= 7 && mode <= 20 && mode != 19)) continue;
            const int grid = 1;
            kern[mode]<<<grid, 128, smem>>>(c, iters, d_out);  // warm
            kern[mode]<<<grid, 128, smem>>>(c, iters, d_out);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) {
                printf("%s: %s\n", c.name, cudaGetErrorString(e));
                return 1;
            }
            unsigned long long h[1024];
            cudaMemcpy(h, d_out, grid * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
            unsigned long long mx = 0;
            for (int i = 0; i < grid; ++i) mx = h[i] > mx ? h[i] : mx;
            const double cyc = (double)mx / iters;  // per MMA (mode >= 7: x batch = latency of a batch)
            const double flop_per_clk = 2.0 * 128 * c.N * 16 / cyc;
            printf("%-42s mode %d: %7.1f cycles/MMA  %7.0f FLOP/clk/SM (floor %d cyc)\n", c.name, mode, cyc,
                   flop_per_clk, 128 * c.N / 256);
            if (mode >= 7 && mode < 14) printf("    batch of %d MMAs + commit + wait: %.0f cycles\n", 1 << (mode - 7), cyc * (1 << (mode - 7)));
        }
    }
    return 0;
}
