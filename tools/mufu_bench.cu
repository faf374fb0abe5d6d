// mufu_bench.cu — MUFU.TANH throughput on this GPU (development aid): every thread runs 8
// independent tanh.approx.f32 chains; reports tanh results per clock per SM for 1..16 warps per SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/mufu_bench tools/mufu_bench.cu
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ float th(float x) { float y; asm volatile("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__global__ void k(float* out, int iters, long long* cyc) {
    float a[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) a[i] = threadIdx.x * 1e-3f + i * 0.1f;
    __syncthreads();
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) a[i] = th(a[i]) * 1.5f;
    }
    __syncthreads();
    long long t1 = clock64();
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < 8; ++i) s += a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    float* out; long long* cyc;
    cudaMalloc(&out, nsm * 1024 * sizeof(float));
    cudaMalloc(&cyc, nsm * sizeof(long long));
    const int iters = 4096;
    for (int warps = 1; warps <= 16; warps *= 2) {
        k<<<nsm, 32 * warps>>>(out, iters, cyc);
        cudaDeviceSynchronize();
        long long c[1024];
        cudaMemcpy(c, cyc, nsm * sizeof(long long), cudaMemcpyDeviceToHost);
        double avg = 0; for (int i = 0; i < nsm; ++i) avg += c[i]; avg /= nsm;
        const double ops = 32.0 * warps * iters * 8;
        printf("warps/SM %2d: %.2f tanh per clock per SM (%.1f cycles per warp-instruction per SMSP)\n", warps, ops / avg,
               avg / (iters * 8.0 * (warps >= 4 ? warps / 4 : 1)));
    }
    return 0;
}
