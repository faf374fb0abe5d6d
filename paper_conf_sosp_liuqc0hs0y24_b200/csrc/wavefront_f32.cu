// wavefront_f32.cu — BK1: the fp32 (TF32 off) correctness path of the wavefront.
//
// Same schedule, flag protocol, segment list and cell-state ring as the tcgen05 path; the gate
// GEMM is plain FP32 FFMA on CUDA cores and the activations use the accurate expf/tanhf
// (fast approximations break the 1e-4 fp32 tolerance).
//
// Persistent cooperative kernel: every CTA walks the global tile sequence (wavefront order,
// ft_common.cuh) with stride gridDim.x.  A tile = (cell, axis, 32 batch rows, 32 hidden units x
// 4 gates).  Thread (u, rg): unit u = tid % 32, rows 4*rg .. 4*rg+3 (rg = tid / 32).
#include <cuda_runtime.h>

#include <cmath>
#include <cstdio>
#include <string>

#include "ft_internal.h"

namespace ft {
namespace {

constexpr int THREADS = 256;
constexpr int BM = F32_BM;    // 32 rows
constexpr int BNU = F32_BNU;  // 32 units
constexpr int KC = 32;        // K chunk

struct F32Smem {
    float a[BM][KC + 1];
    float w[4][KC][BNU];
};

__device__ __forceinline__ const float* src_base(const Tensors& t, int src) {
    return src == SRC_X ? (const float*)t.x : (src == SRC_YS ? (const float*)t.ys : (const float*)t.h_all);
}

__global__ void __launch_bounds__(THREADS)
wavefront_f32_kernel(const __grid_constant__ Problem P, const __grid_constant__ Tensors T) {
    __shared__ F32Smem sm;
    const int tid = threadIdx.x;
    const int u = tid & 31, rg = tid >> 5;
    const int target = flag_target(P);
    Cursor cur = cursor_begin();

    for (long long tile = blockIdx.x; tile < P.ntiles; tile += gridDim.x) {
        const TileId tl = decode_tile(P, cur, tile);
        const Cell& c = tl.cell;
        const int m0 = tl.m * BM, n0 = tl.n * BNU;

        // ---- wait for producer cells (Table 4 dependence vectors) ----------------------
        if (tid == 0) {
            long long prod[3];
            producers(P, c, prod);
            for (int q = 0; q < 3; ++q)
                if (prod[q] >= 0) wait_flag_geq(T.flags + prod[q] * P.MB + tl.m, target);
            __threadfence();
        }
        __syncthreads();

        // ---- z = b + Σ_seg a_seg @ W_seg  (bias first, k ascending, segments in order) ---
        const int n = n0 + u;
        const bool nvalid = n < P.H;
        const int slice_b = (P.kind == KIND_SEQ) ? c.d : c.d * 2 + tl.axis;
        const bool lstm = P.cell == CELL_LSTM;
        const int ng = lstm ? 4 : 1;  // gate blocks of the weight slice (linear cell: one matrix)
        float acc[4][4];
#pragma unroll
        for (int g = 0; g < 4; ++g) {
            const float bv = (nvalid && lstm) ? __ldg(T.b + ((long long)slice_b * 4 + g) * P.H + n) : 0.f;
#pragma unroll
            for (int r = 0; r < 4; ++r) acc[r][g] = bv;
        }
        Segment seg[3];
        segments(P, tl, seg);
        for (int s = 0; s < 3; ++s) {
            if (seg[s].src == SRC_NONE) continue;
            const float* A = src_base(T, seg[s].src);
            const long long arows = src_rows(P, seg[s].src);
            const float* Wt = (const float*)(seg[s].wsel == W_IN ? T.W : T.U);
            const int krows = seg[s].wsel == W_IN ? P.H : u_krows(P);
            for (int k0 = 0; k0 < P.H; k0 += KC) {
                __syncthreads();
                for (int e = tid; e < BM * KC; e += THREADS) {
                    const int r = e / KC, kk = e % KC;
                    const int b = m0 + r, k = k0 + kk;
                    float v = 0.f;
                    if (b < P.B && k < P.H)
                        v = __ldcg(A + ((long long)b * arows + seg[s].row) * P.H + k);
                    sm.a[r][kk] = v;
                }
                for (int e = tid; e < 4 * KC * BNU; e += THREADS) {
                    const int uu = e % BNU, kk = (e / BNU) % KC, g = e / (BNU * KC);
                    const int k = k0 + kk, nn = n0 + uu;
                    float v = 0.f;
                    if (k < P.H && nn < P.H && g < ng)
                        v = __ldg(Wt + (((long long)seg[s].slice * ng + g) * krows + seg[s].krow0 + k) * P.H + nn);
                    sm.w[g][kk][uu] = v;
                }
                __syncthreads();
                const int kend = (P.H - k0) < KC ? (P.H - k0) : KC;
                for (int kk = 0; kk < kend; ++kk) {
                    float a[4], w[4];
#pragma unroll
                    for (int r = 0; r < 4; ++r) a[r] = sm.a[rg * 4 + r][kk];
#pragma unroll
                    for (int g = 0; g < 4; ++g) w[g] = sm.w[g][kk][u];
#pragma unroll
                    for (int r = 0; r < 4; ++r)
#pragma unroll
                        for (int g = 0; g < 4; ++g) acc[r][g] = fmaf(a[r], w[g], acc[r][g]);
                }
            }
        }

        // ---- epilogue: LSTM pointwise update (Listing 2), accurate math -------
        int ci = 0, cj = 0;
        const long long cprod = c_producer(P, tl, &ci, &cj);
        if (cprod >= 0) wait_flag_geq(T.flags + cprod * P.MB + tl.m, target);
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            const int b = m0 + rg * 4 + r;
            if (b >= P.B || !nvalid) continue;
            if (!lstm) {  // Listing 1: y = x@w + s (s = the previous step's output, 0 at t = 0)
                const float sp = (cprod >= 0) ? __ldcg(T.c_ring + c_ring_index(P, c.d, ci, cj, 0, b, n)) : 0.f;
                const float yv = acc[r][0] + sp;
                __stcg((float*)T.h_all + h_all_index(P, c, 0, b, n), yv);
                __stcg(T.c_ring + c_ring_index(P, c.d, c.i, c.j, 0, b, n), yv);
                continue;
            }
            const float ig = 1.f / (1.f + expf(-acc[r][0]));
            const float fg = 1.f / (1.f + expf(-acc[r][1]));
            const float og = 1.f / (1.f + expf(-acc[r][2]));
            const float gh = tanhf(acc[r][3]);
            const float cp = (cprod >= 0) ? __ldcg(T.c_ring + c_ring_index(P, c.d, ci, cj, tl.axis, b, n)) : 0.f;
            const float cn = fg * cp + ig * gh;
            const float hn = og * tanhf(cn);
            __stcg((float*)T.h_all + h_all_index(P, c, tl.axis, b, n), hn);
            __stcg(T.c_ring + c_ring_index(P, c.d, c.i, c.j, tl.axis, b, n), cn);
            if (T.c_all) T.c_all[h_all_index(P, c, tl.axis, b, n)] = cn;
            if (c.d == P.D - 1) ((float*)T.y)[y_index(P, c, tl.axis, b, n)] = hn;
            if (is_last_pos(P, c)) {
                ((float*)T.h_n)[hn_index(P, c, tl.axis, b, n)] = hn;
                T.c_n[hn_index(P, c, tl.axis, b, n)] = cn;
            }
        }
        // ---- publish: this tile's share of the (cell, m-block) readiness counter --------
        __threadfence();
        __syncthreads();
        if (tid == 0) red_release_gpu_add(T.flags + cell_lin(P, c.d, c.i, c.j) * P.MB + tl.m, 1);
    }
}

}  // namespace

cudaError_t launch_wavefront_f32(const Problem& p, const Tensors& t, cudaStream_t s,
                                 std::string* err) {
    int dev = 0, nsm = 0, occ = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (e == cudaSuccess)
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, wavefront_f32_kernel, THREADS, 0);
    if (e != cudaSuccess) {
        if (err) *err = std::string("f32 launch setup: ") + cudaGetErrorString(e);
        return e;
    }
    if (occ < 1) occ = 1;
    long long grid = (long long)nsm * occ;
    if (grid > p.ntiles) grid = p.ntiles;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(THREADS);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    e = cudaLaunchKernelEx(&cfg, wavefront_f32_kernel, p, t);
    if (e == cudaSuccess) set_last_launch("wavefront_f32_kernel grid=" + std::to_string(grid) + " cooperative=1");
    if (e != cudaSuccess && err) *err = std::string("f32 launch: ") + cudaGetErrorString(e);
    return e;
}

}  // namespace ft
