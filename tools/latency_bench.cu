// latency_bench.cu — development microbenchmark (not part of the library): the hardware latencies
// one step of a latency-bound stacked LSTM (C2) cannot avoid, measured on the B200.  Together they
// are the latency roofline of the C2 row: every monotone path from cell (0,0)
// to (D-1,T-1) has T-1 time edges and D-1 depth edges (Table 4), so
//     t_bound = (T-1) * t_time_step + (D-1) * t_depth_hop
// with t_time_step = DSMEM hop + dependent UMMA chain of the recurrent half + TMEM -> registers
//                    + the cell's gate math + issuing the h slice to the cluster (st.async)
// and  t_depth_hop = one release/acquire hand-off through global memory (+ the TMA load of the
//                    64-row operand chunk).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_sosp_liuqc0hs0y24_b200/csrc \
//        -o build/latency_bench tools/latency_bench.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>

#include "ft_sm100.cuh"

using namespace ft;
using namespace ft::sm100;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)
constexpr int N = 512;  // round trips / repetitions

__device__ __forceinline__ uint64_t gt() { return globaltimer_ns(); }

// (1) DSMEM ping-pong between CTA 0 and CTA 1 of a cluster: st.async 16 B + complete_tx on the
//     peer's mbarrier; the peer waits, then answers.  One hop = total / (2N).
__global__ void __cluster_dims__(2, 1, 1) dsmem_pingpong(unsigned long long* out) {
    __shared__ __align__(16) uint4 buf;
    __shared__ uint64_t bar;
    const uint32_t rank = cluster_ctarank(), peer = rank ^ 1;
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbarrier_init();
        mbar_arrive_expect_tx(&bar, 16);  // armed for round 0
    }
    cluster_sync();
    if (threadIdx.x == 0) {
    const uint32_t rbuf = mapa_shared(smem_u32(&buf), peer), rbar = mapa_shared(smem_u32(&bar), peer);
    uint64_t t0 = gt();
    for (int i = 0; i < N; ++i) {
        if (rank == 0) {
            asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %1, %1, %1}, [%2];"
                         ::"r"(rbuf), "r"(i), "r"(rbar) : "memory");
            mbar_wait(&bar, i & 1);
            mbar_arrive_expect_tx(&bar, 16);
        } else {
            mbar_wait(&bar, i & 1);
            mbar_arrive_expect_tx(&bar, 16);
            asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %1, %1, %1}, [%2];"
                         ::"r"(rbuf), "r"(i), "r"(rbar) : "memory");
        }
    }
    if (rank == 0) out[0] = gt() - t0;
    }
    cluster_sync();  // no CTA leaves while its peer may still write into it
}

// (2) global-memory ping-pong between two CTAs on different SMs: red.release.gpu on the peer's
//     counter, ld.acquire.gpu polling on one's own (the depth edge's hand-off).
__global__ void global_pingpong(int* flags, unsigned long long* out) {
    if (threadIdx.x != 0) return;
    const int me = blockIdx.x, peer = me ^ 1;
    uint64_t t0 = gt();
    for (int i = 0; i < N; ++i) {
        if (me == 0) {
            asm volatile("fence.acq_rel.gpu; red.release.gpu.global.add.s32 [%0], 1;" ::"l"(flags + peer) : "memory");
            int v;
            do { asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(flags + me) : "memory"); } while (v < i + 1);
        } else {
            int v;
            do { asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(flags + me) : "memory"); } while (v < i + 1);
            asm volatile("fence.acq_rel.gpu; red.release.gpu.global.add.s32 [%0], 1;" ::"l"(flags + peer) : "memory");
        }
    }
    if (me == 0) out[1] = gt() - t0;
}

// (3) dependent UMMA chain of C2's recurrent half: 16 x M128 N128 K16 (K = H = 256) issued by one
//     elected lane of a converged warp, commit, wait — issue-to-complete latency, averaged.
// (4) TMEM -> registers: 4 x tcgen05.ld 32x32b.x16 (a gate row of 64 accumulator columns) + wait.
// (5) the cell's gate math for U units per thread (bias add, 3 sigmoids + 2 tanh via tanh.approx,
//     c/h update, bf16 pack) as a dependent chain.
template <int U>
__global__ void __launch_bounds__(128, 1) tc_chain(unsigned long long* out, float* sink) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    __shared__ uint64_t bar;
    __shared__ uint32_t slot;
    const int warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbarrier_init();
    }
    if (warp == 0) tmem_alloc(&slot, 256);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = slot;
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0x3c003c00u;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    const uint32_t idesc = make_idesc_bf16_f32(128, 128, false, true);
    const uint64_t ad = make_sdesc(smem_u32(smem), 16, 1024), bd = make_sdesc(smem_u32(smem + 32768), 4096, 512, 4);
    if (warp == 0) {
        uint64_t tot = 0;
        for (int r = 0; r < 64; ++r) {
            __syncwarp();
            const uint64_t t0 = gt();
            if (elect_one()) {
                for (int k = 0; k < 16; ++k)
                    umma_f16(tmem, ad + ((k * 32) >> 4), bd + ((k * 16 * 64) >> 4), idesc, k != 0);
                umma_commit(&bar);
            }
            __syncwarp();
            mbar_wait_warp(&bar, r & 1);
            tc_fence_after();
            if (r >= 8) tot += gt() - t0;
        }
        if (threadIdx.x == 0) out[2] = tot / 56;
    }
    __syncthreads();
    // (4) TMEM loads: warp w reads its lane quadrant
    {
        uint64_t tot = 0;
        float acc = 0.f;
        for (int r = 0; r < 64; ++r) {
            __syncwarp();
            const uint64_t t0 = gt();
            float z[4][16];
#pragma unroll
            for (int g = 0; g < 4; ++g) tmem_ld_32x32b<16>(tmem + ((uint32_t)(warp * 32) << 16) + g * 32, z[g]);
            tmem_wait_ld();
            acc += z[0][r & 15] + z[3][(r + 1) & 15];
            if (r >= 8) tot += gt() - t0;
        }
        if (threadIdx.x == 0) out[3] = tot / 56;
        sink[threadIdx.x] = acc;
    }
    // (5) gate math, U units per thread
    {
        float zi[U], zf[U], zo[U], zg[U], c[U];
#pragma unroll
        for (int u = 0; u < U; ++u) { zi[u] = 0.01f * u; zf[u] = 0.02f * u; zo[u] = -0.01f * u; zg[u] = 0.03f; c[u] = 0.1f; }
        uint64_t tot = 0;
        uint32_t hp = 0;
        for (int r = 0; r < 64; ++r) {
            __syncwarp();
            const uint64_t t0 = gt();
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const float ig = fmaf(0.5f, tanh_approx(fmaf(zi[u], 0.5f, 0.1f)), 0.5f);
                const float fg = fmaf(0.5f, tanh_approx(fmaf(zf[u], 0.5f, 0.2f)), 0.5f);
                const float og = fmaf(0.5f, tanh_approx(fmaf(zo[u], 0.5f, 0.3f)), 0.5f);
                const float gh = tanh_approx(zg[u] + 0.1f);
                c[u] = fmaf(fg, c[u], ig * gh);
                const float h = og * tanh_approx(c[u]);
                hp ^= __float_as_uint(h);
                zi[u] += h;  // a dependency into the next repetition
            }
            __syncwarp();
            if (r >= 8) tot += gt() - t0;
        }
        if (threadIdx.x == 0) out[4] = tot / 56;
        sink[128 + threadIdx.x] = __uint_as_float(hp);
    }
    __syncthreads();
    if (warp == 0) tmem_dealloc(tmem, 256);
}

int main() {
    unsigned long long* d;
    int* flags;
    float* sink;
    CK(cudaMalloc(&d, 16 * 8));
    CK(cudaMalloc(&flags, 64));
    CK(cudaMalloc(&sink, 4096));
    std::vector<unsigned long long> h(16);
    double dsmem = 0, glob = 0;
    for (int rep = 0; rep < 3; ++rep) {
        CK(cudaMemset(flags, 0, 64));
        dsmem_pingpong<<<2, 32>>>(d);
        CK(cudaDeviceSynchronize());
        // the two CTAs of global_pingpong land on different SMs (2 CTAs, large smem each)
        CK(cudaFuncSetAttribute(global_pingpong, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
        global_pingpong<<<2, 32, 200 * 1024>>>(flags, d);
        CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(h.data(), d, 16 * 8, cudaMemcpyDeviceToHost));
        dsmem = h[0] / (2.0 * N);
        glob = h[1] / (2.0 * N);
    }
    CK(cudaFuncSetAttribute(tc_chain<32>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65 * 1024));
    CK(cudaFuncSetAttribute(tc_chain<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65 * 1024));
    tc_chain<32><<<1, 128, 65 * 1024>>>(d, sink);
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(h.data(), d, 16 * 8, cudaMemcpyDeviceToHost));
    const double umma = h[2], tld = h[3], math32 = h[4];
    tc_chain<16><<<1, 128, 65 * 1024>>>(d, sink);
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(h.data(), d, 16 * 8, cudaMemcpyDeviceToHost));
    const double math16 = h[4];
    printf("{\"dsmem_hop_ns\": %.1f, \"global_hop_ns\": %.1f, \"umma_chain_16xM128N128K16_ns\": %.1f, "
           "\"tmem_ld_4x32x32b.x16_ns\": %.1f, \"gate_math_32_units_ns\": %.1f, \"gate_math_16_units_ns\": %.1f}\n",
           dsmem, glob, umma, tld, math32, math16);
    return 0;
}
