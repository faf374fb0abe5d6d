// tma_burst.cu — development microbenchmark (not part of the library): how fast can one SM pull the
// recurrent A operand of a wavefront step into shared memory?  Models one chain step of the bf16
// kernel: NCTA CTAs each own one 16 KB K-chunk (128 rows x 64 bf16, the blocked hb layout);
// round r: every CTA stores its chunk with generic st.global, publishes it (fence + red.release
// on a counter, like the epilogue), then waits for the counter (ld.acquire poll, like the
// activation producer) and TMA-loads NLOAD chunks (its own + others') back to back into NLOAD
// shared-memory slots.  Per CTA and round, %globaltimer stamps: counter seen, each load issued,
// each load landed.  Prints the medians over rounds and CTAs.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/tma_burst tools/tma_burst.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdint>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

constexpr int CHUNK = 16384;   // 128 rows x 128 B
constexpr int MAXL = 12;
constexpr int ROUNDS = 64;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t gtime() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }

__global__ void __launch_bounds__(256, 1) burst(const __grid_constant__ CUtensorMap map, uint8_t* hb, int* flags,
                                                 int nload, int mode, unsigned long long* out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    uint64_t* bars = (uint64_t*)(smem + MAXL * CHUNK);
    const int cta = blockIdx.x, ncta = gridDim.x;
    if (threadIdx.x < MAXL) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bars[threadIdx.x])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncthreads();
    __shared__ uint64_t gtime_seen_s;
    uint64_t& gtime_seen = gtime_seen_s;
    for (int r = 0; r < ROUNDS; ++r) {
        // (1) produce this round's chunk (region r & 1, so round r+1 never overwrites what round r reads)
        uint4* dst = reinterpret_cast<uint4*>(hb + ((size_t)(r & 1) * ncta + cta) * CHUNK);
        for (int i = threadIdx.x; i < CHUNK / 16; i += blockDim.x) dst[i] = make_uint4(r, cta, i, 7);
        __syncthreads();
        if (threadIdx.x == 0) {
            asm volatile("fence.acq_rel.gpu;" ::: "memory");
            asm volatile("red.release.gpu.global.add.s32 [%0], 1;" ::"l"(flags + r), "r"(1) : "memory");
        }
        // (2) consume: wait for every CTA's chunk of round r, then load nload chunks
        if (threadIdx.x == 0) {
            int v;
            do { asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(flags + r) : "memory"); } while (v < ncta);
            gtime_seen = gtime();
            asm volatile("fence.proxy.async.global;" ::: "memory");
            uint64_t t_iss[MAXL];
            if (mode == 4) {  // arm every slot first; the cluster barrier below orders arm before remote writes
                for (int k = 0; k < nload; ++k)
                    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bars[k])), "r"(CHUNK) : "memory");
            }
        }
        if (mode == 4) asm volatile("barrier.cluster.arrive.release.aligned; barrier.cluster.wait.acquire.aligned;" ::: "memory");
        if (mode == 5 && threadIdx.x < 32) {  // every lane k < nload issues load k (one warp-wide TMA instruction)
            __syncwarp();
            const int k = threadIdx.x;
            const uint64_t t_seen = gtime_seen;
            if (k < nload) {
                const int src = (cta + k) % ncta;
                const uint32_t bar = su32(&bars[k]);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(CHUNK) : "memory");
                const int row = ((r & 1) * ncta + src) * 128;
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                    ::"r"(su32(smem + k * CHUNK)), "l"(&map), "r"(0), "r"(row), "r"(bar) : "memory");
            }
            const uint64_t t_i = gtime();
            __syncwarp();
            if (k == 0) {
                uint64_t t_land[MAXL];
                for (int j = 0; j < nload; ++j) {
                    const uint32_t bar = su32(&bars[j]);
                    uint32_t ok = 0;
                    while (!ok)
                        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                                     : "=r"(ok) : "r"(bar), "r"((uint32_t)(r & 1)) : "memory");
                    t_land[j] = gtime();
                }
                unsigned long long* o = out + ((size_t)r * ncta + cta) * (1 + 2 * MAXL);
                o[0] = t_seen;
                for (int j = 0; j < nload; ++j) { o[1 + j] = t_i; o[1 + MAXL + j] = t_land[j]; }
            }
        }
        if (threadIdx.x == 0 && mode != 5) {
            const uint64_t t_seen = gtime_seen;
            uint64_t t_iss[MAXL];
            for (int k = 0; k < nload; ++k) {
                const int src = mode != 1 ? (cta + k) % ncta : k;  // 1: the same chunks on every CTA, else others''
                const uint32_t bar = su32(&bars[k]);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(CHUNK) : "memory");
                const int row = ((r & 1) * ncta + src) * 128;
                if (mode < 2) {
                    asm volatile(
                        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                        ::"r"(su32(smem + k * CHUNK)), "l"(&map), "r"(0), "r"(row), "r"(bar) : "memory");
                } else if (mode == 2) {  // + L2 cache hint (evict_normal), as the kernel's A loads
                    uint64_t pol;
                    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
                    asm volatile(
                        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, %3}], [%4], %5;"
                        ::"r"(su32(smem + k * CHUNK)), "l"(&map), "r"(0), "r"(row), "r"(bar), "l"(pol) : "memory");
                } else if (mode == 4) {  // multicast: cluster of 8; CTA of rank q issues chunk k == q only
                    uint32_t q;
                    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(q));
                    if ((uint32_t)k == q) {
                        const uint16_t mask = 0xFF;
                        asm volatile(
                            "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1, {%2, %3}], [%4], %5;"
                            ::"r"(su32(smem + k * CHUNK)), "l"(&map), "r"(0), "r"(row), "r"(bar), "h"(mask) : "memory");
                    }
                } else {  // the .cta_group::2 form the CTA-pair kernel uses (cluster of 2; own barrier)
                    uint64_t pol;
                    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
                    asm volatile(
                        "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, %3}], [%4], %5;"
                        ::"r"(su32(smem + k * CHUNK)), "l"(&map), "r"(0), "r"(row), "r"(bar), "l"(pol) : "memory");
                }
                t_iss[k] = gtime();
            }
            uint64_t t_land[MAXL];
            for (int k = 0; k < nload; ++k) {
                const uint32_t bar = su32(&bars[k]);
                uint32_t ok = 0;
                while (!ok)
                    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                                 : "=r"(ok) : "r"(bar), "r"((uint32_t)(r & 1)) : "memory");
                t_land[k] = gtime();
            }
            unsigned long long* o = out + ((size_t)r * ncta + cta) * (1 + 2 * MAXL);
            o[0] = t_seen;
            for (int k = 0; k < nload; ++k) { o[1 + k] = t_iss[k]; o[1 + MAXL + k] = t_land[k]; }
        }
        __syncthreads();
    }
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static double med(std::vector<double> v) { std::sort(v.begin(), v.end()); return v.empty() ? 0 : v[v.size() / 2]; }

int main(int argc, char** argv) {
    void* fp = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &fp, 12000, cudaEnableDefault, &q));
    EncFn enc = (EncFn)fp;
    const int ncta_list[] = {16, 144};
    for (int ncta : ncta_list) {
        uint8_t* hb;
        int* flags;
        unsigned long long* out;
        CK(cudaMalloc(&hb, (size_t)2 * ncta * CHUNK));
        CK(cudaMalloc(&flags, ROUNDS * sizeof(int)));
        CK(cudaMalloc(&out, (size_t)ROUNDS * ncta * (1 + 2 * MAXL) * 8));
        CUtensorMap map;
        const cuuint64_t dims[2] = {64, (cuuint64_t)2 * ncta * 128};
        const cuuint64_t str[1] = {128};
        const cuuint32_t box[2] = {64, 128}, es[2] = {1, 1};
        if (enc(&map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, hb, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
            printf("encode failed\n");
            return 1;
        }
        const int smem = MAXL * CHUNK + 1024;
        CK(cudaFuncSetAttribute(burst, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
        const char* names[] = {"others", "same", "hint", "2cta", "mcast8", "lanes"};
        for (int mode : {0, 1, 5})
            for (int nload : {1, 8, 12}) {
                CK(cudaMemset(flags, 0, ROUNDS * sizeof(int)));
                cudaLaunchConfig_t cfg = {};
                cfg.gridDim = dim3(ncta);
                cfg.blockDim = dim3(256);
                cfg.dynamicSmemBytes = smem;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeClusterDimension;
                at[0].val.clusterDim.x = mode == 4 ? 8 : 2;
                at[0].val.clusterDim.y = 1;
                at[0].val.clusterDim.z = 1;
                cfg.attrs = at;
                cfg.numAttrs = 1;
                CK(cudaLaunchKernelEx(&cfg, burst, map, hb, flags, nload, mode, out));
                CK(cudaDeviceSynchronize());
                std::vector<unsigned long long> h((size_t)ROUNDS * ncta * (1 + 2 * MAXL));
                CK(cudaMemcpy(h.data(), out, h.size() * 8, cudaMemcpyDeviceToHost));
                std::vector<double> issue_all, first_land, last_land, per_load;
                for (int r = 4; r < ROUNDS; ++r)
                    for (int c = 0; c < ncta; ++c) {
                        const unsigned long long* o = &h[((size_t)r * ncta + c) * (1 + 2 * MAXL)];
                        issue_all.push_back((o[nload] - o[0]) / 1000.0);
                        first_land.push_back((o[1 + MAXL] - o[0]) / 1000.0);
                        last_land.push_back((o[MAXL + nload] - o[0]) / 1000.0);
                        if (nload > 1) per_load.push_back((o[MAXL + nload] - o[1 + MAXL]) / 1000.0 / (nload - 1));
                    }
                printf("ncta %3d %-6s nload %2d: all issued %.2f us, first landed %.2f us, last landed %.2f us, "
                       "%.3f us per extra load (%.0f GB/s per SM)\n",
                       ncta, names[mode], nload, med(issue_all), med(first_land), med(last_land),
                       med(per_load), nload > 1 ? CHUNK / (med(per_load) * 1e3) : 0.0);
            }
        cudaFree(hb);
        cudaFree(flags);
        cudaFree(out);
    }
    return 0;
}
