// smem_base.cu — prints the shared-window address of the dynamic shared memory base in a plain
// launch and in a 2-CTA cluster launch, and the reserved shared memory per block (development aid
// for reading racecheck reports).
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k() {
    extern __shared__ unsigned char s[];
    if (threadIdx.x == 0)
        printf("block %d: dynamic smem base = 0x%x\n", blockIdx.x, (unsigned)__cvta_generic_to_shared(s));
}
int main() {
    int r = 0;
    cudaDeviceGetAttribute(&r, cudaDevAttrReservedSharedMemoryPerBlock, 0);
    printf("reserved shared memory per block: %d bytes\n", r);
    k<<<1, 32, 1024>>>();
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2);
    cfg.blockDim = dim3(32);
    cfg.dynamicSmemBytes = 1024;
    cudaLaunchAttribute a[1];
    a[0].id = cudaLaunchAttributeClusterDimension;
    a[0].val.clusterDim.x = 2;
    a[0].val.clusterDim.y = 1;
    a[0].val.clusterDim.z = 1;
    cfg.attrs = a;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, k);
    cudaDeviceSynchronize();
    return 0;
}
