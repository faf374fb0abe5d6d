// tma_bench.cu — development microbenchmark: TMA load throughput per SM for different box shapes
// (all loads hit L2: every CTA re-reads the same small tensor).  Not part of the library.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/tma_bench tools/tma_bench.cu
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdint>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int RANK, int STAGES, int NTMA, int HINT = 0, int NPROD = 1>
__global__ void __launch_bounds__(128, 1) tma_loop(const __grid_constant__ CUtensorMap map, int box_bytes, int iters,
                                                   int ncoord, unsigned long long* out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    const int w = threadIdx.x / 32;
    uint8_t* buf = smem + (size_t)w * STAGES * box_bytes * NTMA;
    uint64_t* bars = (uint64_t*)(smem + (size_t)NPROD * STAGES * box_bytes * NTMA) + w * STAGES;
    if (threadIdx.x % 32 == 0 && w < NPROD) {
        for (int s = 0; s < STAGES; ++s)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bars[s])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x % 32 != 0 || w >= NPROD) return;
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    const uint32_t bar0 = su32(&bars[0]);
    const uint32_t buf0 = su32(buf);
    const uint32_t stage_bytes = box_bytes * NTMA;
    long long t0 = clock64();
    int s = 0;
    uint32_t phase = 0;
    int c = (int)(((long long)blockIdx.x * ncoord) / gridDim.x);
    for (int i = 0; i < iters; ++i) {
        const uint32_t bar = bar0 + 8 * s;
        if (i >= STAGES) {
            uint32_t ok = 0;
            while (!ok)
                asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                             : "=r"(ok) : "r"(bar), "r"(phase ^ 1) : "memory");
        }
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(stage_bytes) : "memory");
#pragma unroll
        for (int tt = 0; tt < NTMA; ++tt) {
            const uint32_t dst = buf0 + s * stage_bytes + tt * box_bytes;
            if (RANK == 3 && HINT)
                asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%3, %4, %5}], [%2], %6;"
                             ::"r"(dst), "l"((uint64_t)&map), "r"(bar), "r"(0), "r"(c), "r"(0), "l"(pol) : "memory");
            else if (RANK == 2)
                asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                             ::"r"(dst), "l"((uint64_t)&map), "r"(bar), "r"(0), "r"(c * 256) : "memory");
            else if (RANK == 3)
                asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];"
                             ::"r"(dst), "l"((uint64_t)&map), "r"(bar), "r"(0), "r"(c), "r"(0) : "memory");
            else
                asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];"
                             ::"r"(dst), "l"((uint64_t)&map), "r"(bar), "r"(0), "r"(0), "r"(0), "r"(c) : "memory");
            if (++c == ncoord) c = 0;
        }
        if (++s == STAGES) { s = 0; phase ^= 1; }
    }
    for (int i = 0; i < STAGES; ++i) {  // drain
        const uint32_t bar = bar0 + 8 * s;
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                         : "=r"(ok) : "r"(bar), "r"(phase ^ 1) : "memory");
        if (++s == STAGES) { s = 0; phase ^= 1; }
    }
    if (w == 0) out[blockIdx.x] = clock64() - t0;
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
    void* fp = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &fp, 12000, cudaEnableDefault, &q));
    EncFn enc = (EncFn)fp;
    const size_t bytes = 64ull << 20;
    void* g;
    CK(cudaMalloc(&g, bytes));
    CK(cudaMemset(g, 0, bytes));
    unsigned long long* out;
    CK(cudaMalloc(&out, 148 * sizeof(unsigned long long)));
    int nsm = 148;
    void* big;
    const size_t big_bytes = 2ull << 30;  // 2 GiB: no L2 reuse
    CK(cudaMalloc(&big, big_bytes));
    CK(cudaMemset(big, 1, big_bytes));
    struct Case { const char* name; int rank; cuuint64_t dims[4]; cuuint64_t strides[3]; cuuint32_t box[4]; CUtensorMapSwizzle sw; int ncoord; };
    std::vector<Case> cases = {
        // 2-D K-major operand tile: 64 bf16 (128 B) x 128 rows, rows 2 KB apart
        {"2D 64x128 sw128 (rows 2KB apart)", 2, {1024, 16384}, {2048}, {64, 128}, CU_TENSOR_MAP_SWIZZLE_128B, 16},
        {"2D 64x256 sw128", 2, {1024, 16384}, {2048}, {64, 256}, CU_TENSOR_MAP_SWIZZLE_128B, 16},
        {"2D 64x128 sw128 (rows contiguous 128B)", 2, {64, 262144}, {128}, {64, 128}, CU_TENSOR_MAP_SWIZZLE_128B, 16},
        {"2D 128x64 noswz (256B rows)", 2, {1024, 16384}, {2048}, {128, 64}, CU_TENSOR_MAP_SWIZZLE_NONE, 16},
        {"2D 256x32 noswz (512B rows)", 2, {1024, 16384}, {2048}, {256, 32}, CU_TENSOR_MAP_SWIZZLE_NONE, 16},
        // 3-D activation view (H, rows, B): box (64, 1, 128), batch stride 3.2 MB
        {"3D 64x1x128 sw128 (batch stride 200KB)", 3, {1024, 100, 256}, {2048, 204800}, {64, 1, 128}, CU_TENSOR_MAP_SWIZZLE_128B, 100},
        // 4-D weight view (n, k, gate, slice): box (64, 64, 2, 1)
        {"4D 64x64x2x1 sw128", 4, {1024, 1024, 4, 8}, {2048, 2097152, 8388608}, {64, 64, 2, 1}, CU_TENSOR_MAP_SWIZZLE_128B, 8},
        {"4D 64x64x4x1 sw128", 4, {1024, 1024, 4, 8}, {2048, 2097152, 8388608}, {64, 64, 4, 1}, CU_TENSOR_MAP_SWIZZLE_128B, 8},
    };
    {  // DRAM streaming: 2-D view (64 elems, rows) of the 2 GiB buffer; each CTA streams its own rows
        for (int boxrows : {128, 256}) {
            CUtensorMap m;
            cuuint64_t dims[2] = {64, (cuuint64_t)(big_bytes / 128)};
            cuuint64_t strides[1] = {128};
            cuuint32_t box[2] = {64, (cuuint32_t)boxrows};
            cuuint32_t es[2] = {1, 1};
            CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, big, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                             CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
            if (r != CUDA_SUCCESS) { printf("dram encode failed\n"); return 1; }
            int box_bytes = 128 * boxrows;
            const int iters = 600;  // 600 boxes per CTA
            int ncoord = (int)((big_bytes / 128) / 256 - 1);  // box index c -> rows c*256 (disjoint per CTA)
            for (int stages : {4, 8, 12}) {
                size_t smem = (size_t)stages * box_bytes + 1024;
                if (smem > 227 * 1024) continue;
                void* kfn = stages == 4 ? (void*)tma_loop<2, 4, 1> : stages == 8 ? (void*)tma_loop<2, 8, 1> : (void*)tma_loop<2, 12, 1>;
                CK(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                void* args[] = {&m, &box_bytes, (void*)&iters, &ncoord, &out};
                cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
                cudaEventRecord(e0);
                CK(cudaLaunchKernel(kfn, nsm, 128, args, smem, 0));
                cudaEventRecord(e1);
                CK(cudaDeviceSynchronize());
                float ms; cudaEventElapsedTime(&ms, e0, e1);
                std::vector<unsigned long long> h(148);
                CK(cudaMemcpy(h.data(), out, 148 * 8, cudaMemcpyDeviceToHost));
                double avg = 0; for (auto v : h) avg += v; avg /= 148;
                printf("DRAM stream box %d B stages %2d : %6.1f B/cycle/SM  total %.0f GB/s\n", box_bytes, stages,
                       (double)box_bytes * iters / avg, (double)box_bytes * iters * nsm / (ms * 1e6));
            }
        }
    }
    for (auto& c : cases) {
        CUtensorMap m;
        cuuint32_t es[4] = {1, 1, 1, 1};
        CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, c.rank, g, c.dims, c.strides, c.box, es,
                         CU_TENSOR_MAP_INTERLEAVE_NONE, c.sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) { printf("%-45s encode failed %d\n", c.name, (int)r); continue; }
        int box_bytes = 2;
        for (int i = 0; i < c.rank; ++i) box_bytes *= c.box[i];
        auto run = [&](void* kfn, int ntma, int stages, int nprod = 1, const char* tag = "") -> int {
            const int iters = 4000;
            size_t smem = (size_t)stages * box_bytes * ntma * nprod + 1024;
            if (smem > 227 * 1024) return 0;
            CK(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            void* args[] = {&m, &box_bytes, (void*)&iters, &c.ncoord, &out};
            for (int rep = 0; rep < 2; ++rep) CK(cudaLaunchKernel(kfn, nsm, 128, args, smem, 0));
            CK(cudaDeviceSynchronize());
            std::vector<unsigned long long> h(148);
            CK(cudaMemcpy(h.data(), out, 148 * 8, cudaMemcpyDeviceToHost));
            double avg = 0;
            for (auto v : h) avg += v;
            avg /= 148;
            printf("%-45s%s box %6d B x%d stages %d prod %d : %6.1f B/cycle/SM  (%.0f cycles/stage)\n", c.name, tag, box_bytes, ntma, stages, nprod,
                   (double)box_bytes * ntma * iters * nprod / avg, avg / iters);
            return 0;
        };
#define RUNS(R) run((void*)tma_loop<R, 4, 1>, 1, 4); run((void*)tma_loop<R, 8, 1>, 1, 8); run((void*)tma_loop<R, 4, 2>, 2, 4); run((void*)tma_loop<R, 6, 2>, 2, 6);
        if (c.rank == 2) { RUNS(2) } else if (c.rank == 3) { RUNS(3)
            run((void*)tma_loop<3, 4, 1, 1>, 1, 4, 1, " +hint");
            run((void*)tma_loop<3, 4, 1, 0, 2>, 1, 4, 2, " 2prod");
            run((void*)tma_loop<3, 3, 2, 0, 2>, 2, 3, 2, " 2prod");
        } else { RUNS(4) }
    }
    return 0;
}
