/* c_abi_example.c — the C ABI used from plain C (no Python, no PyTorch): one bf16 stacked-LSTM
 * forward through ft_stacked_lstm_fwd_hostio (host x in, host y / h_n / c_n out; the weights
 * live on the device).  Build:
 *   gcc -O2 -I include examples/c_abi_example.c -L paper_conf_sosp_liuqc0hs0y24_b200 -lft \
 *       -L /usr/local/cuda/lib64 -lcudart -Wl,-rpath,$PWD/paper_conf_sosp_liuqc0hs0y24_b200 -o c_abi_example
 * Run:  ./c_abi_example [batch seq hidden depth]   (prints status, a checksum and timings) */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <cuda_runtime_api.h>

#include "ft.h"

static uint16_t f32_to_bf16(float f) { /* round to nearest even */
    uint32_t u;
    memcpy(&u, &f, 4);
    u += 0x7fffu + ((u >> 16) & 1u);
    return (uint16_t)(u >> 16);
}
static float bf16_to_f32(uint16_t h) {
    uint32_t u = (uint32_t)h << 16;
    float f;
    memcpy(&f, &u, 4);
    return f;
}
static float uniform(uint64_t* s) { /* splitmix64 -> [-1, 1) */
    uint64_t z = (*s += 0x9E3779B97F4A7C15ull);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    z ^= z >> 31;
    return (float)((double)(z >> 11) / 4503599627370496.0 - 1.0);
}

#define CHECK_CUDA(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
    fprintf(stderr, "CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); return 2; } } while (0)

int main(int argc, char** argv) {
    int B = 256, T = 100, H = 1024, D = 16;
    if (argc == 5) { B = atoi(argv[1]); T = atoi(argv[2]); H = atoi(argv[3]); D = atoi(argv[4]); }
    printf("ft_version %d, stacked LSTM B=%d T=%d H=%d D=%d bf16\n", ft_version(), B, T, H, D);
    const size_t nx = (size_t)B * T * H, nw = (size_t)D * 4 * H * H, nb = (size_t)D * 4 * H, ns = (size_t)B * D * H;
    uint16_t *x_h, *y_h, *hn_h, *w_h = malloc(nw * 2), *u_h = malloc(nw * 2);
    float *cn_h, *b_h = malloc(nb * 4);
    CHECK_CUDA(cudaMallocHost((void**)&x_h, nx * 2));   /* pinned: the copies overlap the nest */
    CHECK_CUDA(cudaMallocHost((void**)&y_h, nx * 2));
    CHECK_CUDA(cudaMallocHost((void**)&hn_h, ns * 2));
    CHECK_CUDA(cudaMallocHost((void**)&cn_h, ns * 4));
    uint64_t seed = 42;
    const float scale = 1.0f / sqrtf((float)H);
    for (size_t i = 0; i < nx; ++i) x_h[i] = f32_to_bf16(uniform(&seed));
    for (size_t i = 0; i < nw; ++i) w_h[i] = f32_to_bf16(scale * uniform(&seed));
    for (size_t i = 0; i < nw; ++i) u_h[i] = f32_to_bf16(scale * uniform(&seed));
    for (size_t i = 0; i < nb; ++i) b_h[i] = scale * uniform(&seed);
    void *W, *U, *b, *ws;
    CHECK_CUDA(cudaMalloc(&W, nw * 2));
    CHECK_CUDA(cudaMalloc(&U, nw * 2));
    CHECK_CUDA(cudaMalloc(&b, nb * 4));
    CHECK_CUDA(cudaMemcpy(W, w_h, nw * 2, cudaMemcpyHostToDevice));
    CHECK_CUDA(cudaMemcpy(U, u_h, nw * 2, cudaMemcpyHostToDevice));
    CHECK_CUDA(cudaMemcpy(b, b_h, nb * 4, cudaMemcpyHostToDevice));
    const size_t wsb = ft_stacked_lstm_hostio_workspace_size(B, T, H, D, FT_BF16);
    CHECK_CUDA(cudaMalloc(&ws, wsb));
    cudaStream_t s;
    CHECK_CUDA(cudaStreamCreate(&s));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float ms = 0.f;
    for (int it = 0; it < 4; ++it) { /* warm-up + 3 timed calls */
        if (it == 1) cudaEventRecord(e0, s);
        ft_status st = ft_stacked_lstm_fwd_hostio(B, T, H, D, FT_BF16, x_h, W, U, (const float*)b, y_h, hn_h,
                                                  cn_h, ws, wsb, s);
        if (st != FT_OK) {
            fprintf(stderr, "ft_stacked_lstm_fwd_hostio: %s (%s)\n", ft_status_string(st), ft_last_error());
            return 1;
        }
    }
    cudaEventRecord(e1, s);
    CHECK_CUDA(cudaStreamSynchronize(s));
    cudaEventElapsedTime(&ms, e0, e1);
    double sum = 0.0, asum = 0.0;
    int finite = 1;
    for (size_t i = 0; i < nx; ++i) {
        const float v = bf16_to_f32(y_h[i]);
        finite &= isfinite(v);
        sum += v;
        asum += fabs(v);
    }
    double csum = 0.0;
    for (size_t i = 0; i < ns; ++i) csum += cn_h[i];
    printf("status OK, finite %d, sum(y) %.6f, sum|y| %.6f, sum(c_n) %.6f\n", finite, sum, asum, csum);
    printf("host-buffer forward: %.3f ms per call, %.0f sequences/s\n", ms / 3, B / (ms / 3 / 1e3));
    /* an invalid request is refused before any launch */
    ft_status bad = ft_stacked_lstm_fwd_hostio(B, T, 96, D, FT_BF16, x_h, W, U, (const float*)b, y_h, hn_h, cn_h,
                                               ws, wsb, s);
    printf("hidden=96 (not a multiple of 64): %s\n", ft_status_string(bad));
    return finite && bad == FT_ERR_UNSUPPORTED ? 0 : 1;
}
