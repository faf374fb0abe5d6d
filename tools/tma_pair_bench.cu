// tma_pair_bench.cu — development microbenchmark: TMA throughput under the CTA-pair protocol of the
// wavefront kernel (.cta_group::2 loads completing on the leader's mbarrier; the leader hands the
// slot back to the peer with a remote arrive).  L2-resident data.  Not part of the library.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t r) { uint32_t o; asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(o) : "r"(a), "r"(r)); return o; }
__device__ __forceinline__ void wait(uint32_t bar, uint32_t par) {
    uint32_t ok = 0;
    while (!ok) asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }" : "=r"(ok) : "r"(bar), "r"(par) : "memory");
}
template <int STAGES, int NBOX, int PAIR>
__global__ void __launch_bounds__(128, 1) pair_loop(const __grid_constant__ CUtensorMap map, int box_bytes, int iters, unsigned long long* out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    uint64_t* full = (uint64_t*)(smem + (size_t)STAGES * box_bytes * NBOX);
    uint64_t* empty = full + STAGES;
    uint32_t rank = 0;
    if (PAIR) asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&empty[s])));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (PAIR) asm volatile("barrier.cluster.arrive.release.aligned; barrier.cluster.wait.acquire.aligned;" ::: "memory");
    long long t0 = clock64();
    if (threadIdx.x == 0) {
        const uint32_t full0 = PAIR ? mapa(su32(full), 0) : su32(full);
        int s = 0; uint32_t ph = 0;
        for (int i = 0; i < iters; ++i) {
            wait(su32(&empty[s]), ph ^ 1);
            if (rank == 0) asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(box_bytes * NBOX * (PAIR ? 2 : 1)) : "memory");
            for (int b = 0; b < NBOX; ++b) {
                const uint32_t dst = su32(smem + ((size_t)s * NBOX + b) * box_bytes);
                const int c = (int)((blockIdx.x * 3 + i + b) % 16) * 128 + (int)rank * 64;
                if (PAIR)
                    asm volatile("cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                                 ::"r"(dst), "l"((uint64_t)&map), "r"(full0 + 8 * s), "r"(0), "r"(c) : "memory");
                else
                    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                                 ::"r"(dst), "l"((uint64_t)&map), "r"(full0 + 8 * s), "r"(0), "r"(c) : "memory");
            }
            if (++s == STAGES) { s = 0; ph ^= 1; }
        }
    } else if (threadIdx.x == 32 && rank == 0) {  // consumer: wait full, hand the slot back to both CTAs
        int s = 0; uint32_t ph = 0;
        for (int i = 0; i < iters; ++i) {
            wait(su32(&full[s]), ph);
            if (PAIR) {
                asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(mapa(su32(&empty[s]), 0)) : "memory");
                asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(mapa(su32(&empty[s]), 1)) : "memory");
            } else {
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[s])) : "memory");
            }
            if (++s == STAGES) { s = 0; ph ^= 1; }
        }
        out[blockIdx.x] = clock64() - t0;
    }
    __syncthreads();
    if (PAIR) asm volatile("barrier.cluster.arrive.release.aligned; barrier.cluster.wait.acquire.aligned;" ::: "memory");
}
typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int main() {
    void* fp = nullptr; cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &fp, 12000, cudaEnableDefault, &q));
    EncFn enc = (EncFn)fp;
    void* g; CK(cudaMalloc(&g, 64 << 20)); CK(cudaMemset(g, 0, 64 << 20));
    unsigned long long* out; CK(cudaMalloc(&out, 148 * 8)); CK(cudaMemset(out, 0, 148 * 8));
    CUtensorMap m; cuuint64_t dims[2] = {64, 65536}; cuuint64_t st[1] = {128}; cuuint32_t box[2] = {64, 128}; cuuint32_t es[2] = {1, 1};
    if (enc(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, g, dims, st, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) { printf("enc fail\n"); return 1; }
    int box_bytes = 16384, iters = 4000;
    auto run = [&](void* k, int pair, int nbox, int stages, const char* name) -> int {
        size_t smem = (size_t)stages * box_bytes * nbox + 1024;
        CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        cudaLaunchConfig_t cfg = {}; cfg.gridDim = dim3(148); cfg.blockDim = dim3(128); cfg.dynamicSmemBytes = smem;
        cudaLaunchAttribute at[1]; at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = pair ? 2 : 1; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
        cfg.attrs = at; cfg.numAttrs = 1;
        void* args[] = {&m, &box_bytes, &iters, &out};
        for (int r = 0; r < 2; ++r) CK(cudaLaunchKernelExC(&cfg, k, args));
        CK(cudaDeviceSynchronize());
        std::vector<unsigned long long> h(148); CK(cudaMemcpy(h.data(), out, 148 * 8, cudaMemcpyDeviceToHost));
        double avg = 0; int n = 0; for (auto v : h) if (v) { avg += v; ++n; } avg /= n;
        printf("%-28s boxes/stage %d stages %d : %6.0f cycles/stage  %6.1f B/cycle/CTA\n", name, nbox, stages, avg / iters, (double)box_bytes * nbox * iters / avg);
        return 0;
    };
    run((void*)pair_loop<6, 2, 0>, 0, 2, 6, "single CTA");
    run((void*)pair_loop<6, 2, 1>, 1, 2, 6, "CTA pair (.cta_group::2)");
    run((void*)pair_loop<6, 1, 1>, 1, 1, 6, "CTA pair (.cta_group::2)");
    run((void*)pair_loop<3, 4, 1>, 1, 4, 3, "CTA pair (.cta_group::2)");
    return 0;
}
