// ft_internal.h — declarations shared by the library's translation units (not installed).
#pragma once

#include <cuda_runtime.h>

#include <cstdlib>
#include <string>
#include <utility>

#include "ft_common.cuh"

namespace ft {

// Environment knobs (every one is documented in include/ft.h; none changes a result beyond the
// summation-order freedom that header states).  Read per call, so a test can flip them.
inline const char* env_str(const char* name) { return getenv(name); }
inline bool env_off(const char* name) {  // set to "0"
    const char* e = getenv(name);
    return e && e[0] == '0' && e[1] == 0;
}
inline bool env_flag(const char* name) {  // set and not "0"
    const char* e = getenv(name);
    return e && e[0] && !(e[0] == '0' && e[1] == 0);
}

// Device pointers of one call.  `y` is `out` for the grid call.
struct Tensors {
    const void* x = nullptr;
    const void* ys = nullptr;
    const void* W = nullptr;
    const void* U = nullptr;
    const float* b = nullptr;
    void* y = nullptr;
    void* h_n = nullptr;
    float* c_n = nullptr;
    void* h_all = nullptr;   // f32 path: never NULL at launch (workspace stand-in); bf16: optional
    void* hb = nullptr;      // bf16 path: blocked SSA activations [h_rows][H/64][Bp][64] (workspace)
    void* xb = nullptr;      // bf16 path: x packed into the same blocked layout [L0][H/64][Bp][64]
    void* yb = nullptr;      // bf16 grid: ys packed [L1][H/64][Bp][64]
    float* c_all = nullptr;  // optional
    float* c_ring = nullptr; // workspace: fp32 cell-state ring
    int* flags = nullptr;    // workspace: readiness counters [ncells][MB]
    // host-IO overlap (ft_stacked_lstm_fwd_hostio): the bf16 streaming kernel adds 1 to
    // ysig[t / ychunk] per epilogue warp once its part of y(·, t, ·) is stored and fenced, so a
    // copy stream can move finished time chunks of y to the host while the nest still runs.
    // host-IO overlap of x: x arrives in time chunks from the host (a copy stream sets
    // xsig[c] = 1 after chunk c); the streaming kernel then reads layer-0 inputs straight from
    // x [B][T][H] (3-D TMA, no pack) and waits for xsig[t / xchunk] before a chunk's first use.
    int* xsig = nullptr;
    int xchunk = 0;
    int* ysig = nullptr;
    int ychunk = 0;
    int* ysig_per_step = nullptr;  // HOST: set by the launcher to the increments per time step
                                   // (0 = this launch does not signal; copy y after the kernel)
    // host-IO overlap of the final states: after storing its share of h_n / c_n (cell (d, T-1)),
    // every epilogue warp fences at system scope and adds 1 to nsig[d]; a second copy stream
    // moves layer d's rows to the host once nsig[d] reaches *ysig_per_step (same count per cell)
    int* nsig = nullptr;
    int* nsig0_per_step = nullptr; // HOST: nsig[0]'s count when layer 0 runs narrower slabs (owner
                                   // mode 3 of dilated nests; the host-buffer call itself takes
                                   // stacked nests); 0 = *ysig_per_step
    int* ysig_per_chunk = nullptr; // HOST: 1 = owner walk: each warp signals once per chunk (its
                                   // last step of the chunk), so a chunk completes at per_step
};

// Text of the last forward launch on this thread (ft_last_launch): kernel, grid and schedule.
void set_last_launch(const std::string& s);

// Persistent cluster launch.  The cluster grid is sized by cudaOccupancyMaxActiveClusters, so on
// an otherwise idle device every CTA is resident at once.  (The cooperative attribute next to the
// cluster dimension was tried: the driver accepts it, but Nsight Compute's kernel replay then
// fails with LaunchFailed, so it is not used.)  Launches of this library on one device are
// ordered one after another (ft_api.cu PersistentOrder), so two of its persistent kernels never
// split the SMs; another application's kernel can only delay CTAs until it finishes.
template <typename... KArgs, typename... Args>
cudaError_t launch_cluster_persistent(cudaLaunchConfig_t cfg, const cudaLaunchAttribute* base, int nbase,
                                      int* cooperative, void (*kernel)(KArgs...), Args&&... args) {
    cfg.attrs = const_cast<cudaLaunchAttribute*>(base);
    cfg.numAttrs = nbase;
    if (cooperative) *cooperative = 0;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

// Tile shapes of the two kernels.
constexpr int F32_BM = 32, F32_BNU = 32;     // SIMT correctness path (BK1)
constexpr int BF16_BM = 128, BF16_BNU = 64;  // tcgen05 path (BK2–BK4)

// Number of fp32 ring elements the cell state needs.
long long c_ring_elems(const Problem& p);

int l2_persist_mib();  // ft_set_l2_persist setting (-1 auto, 0 off, else MiB)
cudaError_t launch_wavefront_f32(const Problem& p, const Tensors& t, cudaStream_t s,
                                 std::string* err);
cudaError_t launch_wavefront_bf16(const Problem& p, const Tensors& t, cudaStream_t s,
                                  std::string* err);
// which bf16 kernel launch_wavefront_bf16 runs for `p`: 0 DSMEM cluster, 1 SMEM-resident,
// 2 streaming (the only one that honours Tensors::xsig / ysig)
int bf16_kernel_choice(const Problem& p);
// NEXT-4 back-to-back GEMMs (b2b_gemm.cu): D[M][64] = (A[M][64] @ B[64][N]) @ C[N][64]
cudaError_t launch_b2b_gemm(int M, int N, const void* A, const void* B, const void* C, float* D,
                            cudaStream_t s, std::string* err);
// a6: whether a bf16 stacked / dilated LSTM keeps hb as per-layer rings (p.hring): every problem
// the streaming kernel runs — i.e. not one of the small SMEM-resident / DSMEM-cluster shapes,
// which keep one hb row per (d, t)
bool hb_ring_eligible(const Problem& p);
// a5 weight-resident mode (wavefront_resident.cu): slab width 16/32 when the weights fit, else 0
int resident_bnu(const Problem& p, int nsm);
bool cluster_kernel_applies(const Problem& p);
cudaError_t launch_wavefront_cluster(const Problem& p, const Tensors& t, cudaStream_t s, std::string* err);
cudaError_t launch_wavefront_resident(const Problem& p, const Tensors& t, cudaStream_t s, int bnu,
                                      std::string* err);

// NEXT-2 layer-sequential comparison schedule (layerwise.cu): per layer a hoisted input
// projection GEMM (cuBLAS) + a U-resident recurrent kernel.
int layerwise_supported(int B, int H, int nsm, std::string* why);
size_t layerwise_ws_bytes(int B, int T, int H);
cudaError_t launch_layerwise(int B, int T, int H, int D, const void* x, const void* W, const void* U,
                             const float* b, void* y, void* h_n, float* c_n, void* h_all,
                             float* c_all, void* ws, cudaStream_t s, std::string* err);

}  // namespace ft
