// ft_api.cu — the C ABI (include/ft.h): argument validation, workspace planning, problem
// construction and kernel dispatch.  No compute happens here; every step of the path runs in
// the kernels of wavefront_f32.cu / wavefront_bf16.cu.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <string>
#include <mutex>
#include <algorithm>
#include <cuda.h>

#include "../../include/ft.h"
#include "ft_internal.h"

#define FT_API extern "C" __attribute__((visibility("default")))

namespace {

thread_local std::string g_last_error = "no error";
thread_local std::string g_last_launch = "none";

ft_status fail(ft_status s, const std::string& msg) {
    g_last_error = msg;
    return s;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

size_t round_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

size_t elem_size(ft_dtype dt) { return dt == FT_BF16 ? 2 : 4; }

// Build the launch problem; returns OK or INVALID/UNSUPPORTED with g_last_error set.
ft_status make_problem(int kind, int B, int L0, int L1, int H, int D, const int* dil,
                       ft_dtype dt, ft::Problem* p, int cell = ft::CELL_LSTM) {
    if (dt != FT_F32 && dt != FT_BF16) return fail(FT_ERR_INVALID_ARGUMENT, "unknown dtype");
    if (B <= 0 || L0 <= 0 || L1 <= 0 || H <= 0 || D <= 0)
        return fail(FT_ERR_INVALID_ARGUMENT, "every dimension must be > 0");
    if (D > FT_MAX_DEPTH) return fail(FT_ERR_UNSUPPORTED, "depth > FT_MAX_DEPTH");
    if (kind == ft::KIND_SEQ) {
        if (!dil) return fail(FT_ERR_INVALID_ARGUMENT, "dilations is NULL");
        for (int d = 0; d < D; ++d)
            if (dil[d] < 1) return fail(FT_ERR_INVALID_ARGUMENT, "dilation < 1");
    }
    if (dt == FT_BF16 && H % 64 != 0)
        return fail(FT_ERR_UNSUPPORTED, "bf16 path requires hidden % 64 == 0");
    // 32-bit coordinate / index guards (TMA coordinates and row indices are int32)
    const long long rows = (kind == ft::KIND_SEQ) ? (long long)D * L0 : (long long)D * L0 * L1 * 2;
    if (rows > (1ll << 30) || (long long)B > (1ll << 30) || (long long)H > (1 << 20))
        return fail(FT_ERR_UNSUPPORTED, "problem too large for 32-bit coordinates");

    std::memset(p, 0, sizeof(*p));
    p->kind = kind;
    p->cell = cell;
    p->B = B;
    p->H = H;
    p->D = D;
    p->L0 = L0;
    p->L1 = L1;
    p->naxes = (kind == ft::KIND_SEQ) ? 1 : 2;
    // bf16: one tcgen05 tile covers 128 batch rows (1 CTA) or 256 (a CTA pair, cta_group::2)
    p->BM = dt == FT_BF16 ? (B > ft::BF16_BM ? 2 * ft::BF16_BM : ft::BF16_BM) : ft::F32_BM;
    p->flag_mult = dt == FT_BF16 ? p->BM / ft::BF16_BM : 1;
    {
        // a5 weight residency: when every layer's weights fit in about half of the 126 MB L2
        // they are kept there across time steps (EVICT_LAST); otherwise they stream (EVICT_FIRST)
        // — a 256 MiB weight set cannot be resident, each diagonal re-reads it.
        const double wbytes =
            cell == ft::CELL_LINEAR
                ? (double)D * H * H * (dt == FT_BF16 ? 2 : 4)
                : (double)D * p->naxes * 4.0 * H * ((double)H + (kind == ft::KIND_SEQ ? H : 2.0 * H)) *
                      (dt == FT_BF16 ? 2 : 4);
        p->resident_layers = wbytes <= 64.0 * 1024 * 1024 ? D : 0;
        p->persist_layers = -1;  // -1: sized by ft_set_l2_persist
        p->debug = 0;
#ifdef FT_DEV_EXPERIMENTS  // development builds only (tools/variant_build.sh); never in libft.so
        if (const char* env = getenv("FT_L2_RESIDENT_LAYERS")) p->resident_layers = atoi(env);
        if (const char* pe = getenv("FT_L2_PERSIST_LAYERS")) p->persist_layers = atoi(pe);
        if (const char* dbg = getenv("FT_DEBUG")) p->debug = atoi(dbg);  // results INVALID
#endif
        // documented schedule knob (include/ft.h): random delays before every counter release;
        // results are unchanged, the tests use it to shake out ordering bugs
        if (ft::env_flag("FT_STRESS")) p->debug |= 64;
    }
    p->BNU = dt == FT_BF16 ? ft::BF16_BNU : ft::F32_BNU;
    if (cell == ft::CELL_LINEAR && dt == FT_BF16) p->BNU = 4 * ft::BF16_BNU;  // 256 units per tile
    p->MB = (B + p->BM - 1) / p->BM;
    p->NT = (H + p->BNU - 1) / p->BNU;
    p->ncells = (long long)D * L0 * L1;
    p->ntiles = p->ncells * p->naxes * p->MB * p->NT;
    if (kind == ft::KIND_SEQ) {
        int off = 0;
        for (int d = 0; d < D; ++d) {
            p->dil[d] = dil[d];
            p->ring_off[d] = off;
            const long long len = dil[d] < L0 ? dil[d] : L0;  // one slot per residue of t mod s_d
            off += (int)len;
        }
        p->ring_off[D] = off;
        // a6 for the bf16 streaming kernel: the SSA buffer hb as per-layer rings (ft_common.cuh
        // hb_slot_row) plus two T-step regions for band-boundary layers — C3: 1600 rows of
        // (d, t) → 16·4 + 200.  The launcher lays the slots out once the band is known.
        if (dt == FT_BF16 && cell == ft::CELL_LSTM && ft::hb_ring_eligible(*p) && !ft::env_off("FT_SSA_RING")) {
            long long rows = 2ll * L0;
            for (int d = 0; d < D; ++d) rows += ft::hb_ring_len(dil[d], L0);
            if (rows < (long long)D * L0) {
                p->hring = 1;
                p->hb_rows = (int)rows;
                ft::hb_layout(*p, 0);  // the paper order's layout; the launcher redoes it per band
            }
        }
    }
    // bf16: TMA row coordinates into the blocked buffers are int32
    if (dt == FT_BF16 && (ft::hb_rows_total(*p) >= (1ll << 31) ||
                          (long long)L0 * (H / 64) * p->MB * p->BM >= (1ll << 31)))
        return fail(FT_ERR_UNSUPPORTED, "problem too large: blocked activation rows exceed int32 TMA coordinates");
    return FT_OK;
}

struct WsPlan {
    size_t flags_off, flags_bytes;
    size_t ring_off, ring_bytes;
    size_t hall_off, hall_bytes;
    size_t xb_off, xb_bytes, yb_off, yb_bytes;  // bf16: inputs packed into the blocked layout
    size_t total;
};

WsPlan plan_workspace(const ft::Problem& p, ft_dtype dt, bool h_all_provided) {
    WsPlan w{};
    w.flags_off = 0;
    // readiness counters: [2][ncells][MB] (h-ready, c-ready: ft_common.cuh cflag_index)
    const size_t nflags = 2 * (size_t)p.ncells * p.MB;
    w.flags_bytes = round_up(nflags * sizeof(int), 256);
    w.ring_off = w.flags_off + w.flags_bytes;
    w.ring_bytes = round_up((size_t)ft::c_ring_elems(p) * sizeof(float), 256);
    w.hall_off = w.ring_off + w.ring_bytes;
    if (dt == FT_BF16)  // the blocked SSA activation buffer (full, or per-layer rings: p.hring)
        w.hall_bytes = round_up((size_t)ft::hb_rows_total(p) * 64 * 2, 256);
    else
        w.hall_bytes = h_all_provided
                           ? 0
                           : round_up((size_t)p.B * ft::h_rows(p) * p.H * elem_size(dt), 256);
    w.xb_off = w.hall_off + w.hall_bytes;
    w.xb_bytes = dt == FT_BF16 ? round_up((size_t)p.L0 * p.H * ((size_t)p.MB * p.BM) * 2, 256) : 0;
    w.yb_off = w.xb_off + w.xb_bytes;
    w.yb_bytes = (dt == FT_BF16 && p.kind == ft::KIND_GRID)
                     ? round_up((size_t)p.L1 * p.H * ((size_t)p.MB * p.BM) * 2, 256)
                     : 0;
    w.total = w.yb_off + w.yb_bytes;
    return w;
}

ft_status check_device() {
    int dev = 0, major = 0, minor = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
    if (e != cudaSuccess) return fail(FT_ERR_CUDA, std::string("no usable CUDA device: ") + cudaGetErrorString(e));
    if (major != 10 || minor != 0)
        return fail(FT_ERR_UNSUPPORTED, "this library is built for sm_100a (B200) only; device is sm_" +
                                            std::to_string(major) + std::to_string(minor));
    return FT_OK;
}

// Co-residency of persistent launches.  The wavefront kernels spin on each other's CTAs, so all
// CTAs of one launch must be resident together.  A single launch guarantees that by construction
// (cooperative launch, or a cluster grid sized by cudaOccupancyMaxActiveClusters), but two of the
// library's launches on two streams of one device could split the SMs between them and both spin.
// So every persistent launch of this process on a device is ordered after the previous one: the
// caller's stream waits on an event recorded after the previous launch (no host blocking; the
// streams stay otherwise independent).  Skipped while the stream is being captured into a graph
// (the graph's own launch order applies).  Processes without MPS never run kernels concurrently.
class PersistentOrder {
  public:
    explicit PersistentOrder(cudaStream_t s) : s_(s) {
        cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
        if (cudaStreamIsCapturing(s, &cs) != cudaSuccess) {
            cudaGetLastError();
            return;
        }
        if (cs != cudaStreamCaptureStatusNone) return;
        int dev = 0;
        if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return;
        lock_ = std::unique_lock<std::mutex>(mu());
        cudaEvent_t& ev = last()[dev];
        if (!ev && cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess) {
            cudaGetLastError();
            ev = nullptr;
            lock_.unlock();
            return;
        }
        ev_ = ev;
        if (used()[dev] && cudaStreamWaitEvent(s, ev, 0) != cudaSuccess) cudaGetLastError();
        used()[dev] = true;
    }
    ~PersistentOrder() {
        if (ev_ && cudaEventRecord(ev_, s_) != cudaSuccess) cudaGetLastError();
    }

  private:
    static std::mutex& mu() { static std::mutex m; return m; }
    static cudaEvent_t* last() { static cudaEvent_t e[64] = {}; return e; }
    static bool* used() { static bool u[64] = {}; return u; }
    cudaStream_t s_;
    cudaEvent_t ev_ = nullptr;
    std::unique_lock<std::mutex> lock_;
};

ft_status run(const ft::Problem& p, ft_dtype dt, ft::Tensors t, void* workspace,
              size_t workspace_bytes, void* stream) {
    const WsPlan w = plan_workspace(p, dt, t.h_all != nullptr);
    if (w.total > 0 && !workspace) return fail(FT_ERR_INVALID_ARGUMENT, "workspace is NULL");
    if (workspace && !aligned16(workspace))
        return fail(FT_ERR_INVALID_ARGUMENT, "workspace not 16-byte aligned");
    if (workspace_bytes < w.total)
        return fail(FT_ERR_WORKSPACE_TOO_SMALL,
                    "workspace_bytes " + std::to_string(workspace_bytes) + " < required " +
                        std::to_string(w.total));
    ft_status st = check_device();
    if (st != FT_OK) return st;
    uint8_t* ws = static_cast<uint8_t*>(workspace);
    t.flags = reinterpret_cast<int*>(ws + w.flags_off);
    t.c_ring = reinterpret_cast<float*>(ws + w.ring_off);
    if (dt == FT_BF16) {
        t.hb = ws + w.hall_off;
        t.xb = ws + w.xb_off;
        t.yb = w.yb_bytes ? ws + w.yb_off : nullptr;
    } else if (!t.h_all)
        t.h_all = ws + w.hall_off;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    PersistentOrder order(s);
    cudaError_t e = cudaMemsetAsync(t.flags, 0, w.flags_bytes, s);  // BK0: reset readiness flags
    if (e != cudaSuccess) return fail(FT_ERR_CUDA, std::string("flag reset: ") + cudaGetErrorString(e));
    std::string err;
    e = (dt == FT_BF16) ? ft::launch_wavefront_bf16(p, t, s, &err)
                        : ft::launch_wavefront_f32(p, t, s, &err);
    if (e != cudaSuccess) return fail(FT_ERR_CUDA, err.empty() ? cudaGetErrorString(e) : err);
    return FT_OK;
}

#define REQUIRE_PTR(ptr, name)                                                               \
    do {                                                                                     \
        if (!(ptr)) return fail(FT_ERR_INVALID_ARGUMENT, std::string(name) + " is NULL");    \
        if (!aligned16(ptr))                                                                 \
            return fail(FT_ERR_INVALID_ARGUMENT, std::string(name) + " not 16-byte aligned"); \
    } while (0)
#define OPTIONAL_PTR(ptr, name)                                                              \
    do {                                                                                     \
        if ((ptr) && !aligned16(ptr))                                                        \
            return fail(FT_ERR_INVALID_ARGUMENT, std::string(name) + " not 16-byte aligned"); \
    } while (0)

ft_status seq_fwd(int batch, int seq, int hidden, int depth, const int* dil, ft_dtype dt,
                  const void* x, const void* W, const void* U, const float* b, void* y,
                  void* h_n, float* c_n, void* h_all, float* c_all, void* workspace,
                  size_t workspace_bytes, void* stream) {
    ft::Problem p;
    ft_status st = make_problem(ft::KIND_SEQ, batch, seq, 1, hidden, depth, dil, dt, &p);
    if (st != FT_OK) return st;
    REQUIRE_PTR(x, "x");
    REQUIRE_PTR(W, "W");
    REQUIRE_PTR(U, "U");
    REQUIRE_PTR(b, "b");
    REQUIRE_PTR(y, "y");
    REQUIRE_PTR(h_n, "h_n");
    REQUIRE_PTR(c_n, "c_n");
    OPTIONAL_PTR(h_all, "h_all");
    OPTIONAL_PTR(c_all, "c_all");
    ft::Tensors t;
    t.x = x;
    t.W = W;
    t.U = U;
    t.b = b;
    t.y = y;
    t.h_n = h_n;
    t.c_n = c_n;
    t.h_all = h_all;
    t.c_all = c_all;
    return run(p, dt, t, workspace, workspace_bytes, stream);
}

}  // namespace

namespace ft {
static int g_l2_persist_mib = 0;  // ft_set_l2_persist: 0 off (default), -1 auto, else MiB
int l2_persist_mib() { return g_l2_persist_mib; }
void set_last_error(const std::string& msg) { g_last_error = msg; }
void set_last_launch(const std::string& s) { g_last_launch = s; }
long long c_ring_elems(const Problem& p) {
    if (p.kind == KIND_SEQ) return (long long)p.ring_off[p.D] * c_slot_elems(p);
    return ((long long)p.D * p.L1 + (long long)p.D * p.L0) * c_slot_elems(p);
}
}  // namespace ft

FT_API int ft_version(void) { return FT_VERSION; }

FT_API const char* ft_last_launch(void) { return g_last_launch.c_str(); }

FT_API ft_status ft_set_l2_persist(int mib) {
    if (mib < -1) return fail(FT_ERR_INVALID_ARGUMENT, "ft_set_l2_persist: mib must be >= -1");
    ft::g_l2_persist_mib = mib;
    return FT_OK;
}

FT_API const char* ft_status_string(ft_status s) {
    switch (s) {
        case FT_OK: return "FT_OK";
        case FT_ERR_INVALID_ARGUMENT: return "FT_ERR_INVALID_ARGUMENT";
        case FT_ERR_UNSUPPORTED: return "FT_ERR_UNSUPPORTED";
        case FT_ERR_CUDA: return "FT_ERR_CUDA";
        case FT_ERR_NCCL: return "FT_ERR_NCCL";
        case FT_ERR_WORKSPACE_TOO_SMALL: return "FT_ERR_WORKSPACE_TOO_SMALL";
    }
    return "FT_ERR_UNKNOWN";
}

FT_API const char* ft_last_error(void) { return g_last_error.c_str(); }

FT_API size_t ft_stacked_lstm_workspace_size(int batch, int seq, int hidden, int depth, ft_dtype dt,
                                             int h_all_provided) {
    if (depth <= 0 || depth > FT_MAX_DEPTH) return 0;
    int ones[FT_MAX_DEPTH];
    for (int d = 0; d < depth; ++d) ones[d] = 1;
    ft::Problem p;
    if (make_problem(ft::KIND_SEQ, batch, seq, 1, hidden, depth, ones, dt, &p) != FT_OK) return 0;
    return plan_workspace(p, dt, h_all_provided != 0).total;
}

FT_API ft_status ft_stacked_lstm_fwd(int batch, int seq, int hidden, int depth, ft_dtype dt,
                                     const void* x, const void* W, const void* U, const float* b,
                                     void* y, void* h_n, float* c_n, void* h_all, float* c_all,
                                     void* workspace, size_t workspace_bytes, void* stream) {
    if (depth <= 0) return fail(FT_ERR_INVALID_ARGUMENT, "every dimension must be > 0");
    if (depth > FT_MAX_DEPTH) return fail(FT_ERR_UNSUPPORTED, "depth > FT_MAX_DEPTH");
    int ones[FT_MAX_DEPTH];
    for (int d = 0; d < depth; ++d) ones[d] = 1;
    return seq_fwd(batch, seq, hidden, depth, ones, dt, x, W, U, b, y, h_n, c_n, h_all, c_all,
                   workspace, workspace_bytes, stream);
}

namespace {
// time steps per host-IO chunk (x in, y out): 5 measured best at C3 (exposed copy time per
// step 0.35 ms vs 0.40 ms at 10 and 0.46 ms at 3, profiles/r2_ab_hostio_chunk.txt);
// FT_HOSTIO_CHUNK overrides (experiments)
int hostio_chunk() {
    const char* e = getenv("FT_HOSTIO_CHUNK");
    const int c = e ? atoi(e) : 5;
    return c >= 1 ? c : 5;
}

struct HostIoPlan {
    size_t x_off, y_off, hn_off, cn_off, ysig_off, xsig_off, nsig_off, inner_off, total;
    int nchunks;
};
HostIoPlan plan_hostio(int batch, int seq, int hidden, int depth, ft_dtype dt, size_t inner) {
    const size_t es = elem_size(dt);
    HostIoPlan h{};
    h.nchunks = seq;  // room for chunks of 1 step; a call uses ceil(seq / hostio_chunk())
    h.x_off = 0;
    h.y_off = round_up((size_t)batch * seq * hidden * es, 256);
    h.hn_off = h.y_off + round_up((size_t)batch * seq * hidden * es, 256);
    h.cn_off = h.hn_off + round_up((size_t)batch * depth * hidden * es, 256);
    h.ysig_off = h.cn_off + round_up((size_t)batch * depth * hidden * 4, 256);
    h.xsig_off = h.ysig_off + round_up((size_t)h.nchunks * sizeof(int), 256);
    h.nsig_off = h.xsig_off + round_up((size_t)h.nchunks * sizeof(int), 256);
    h.inner_off = h.nsig_off + round_up((size_t)depth * sizeof(int), 256);
    h.total = h.inner_off + inner;
    return h;
}

// Per-device copy stream of the host-IO overlap, created once (it lives as long as the process's
// CUDA context; concurrent calls may share it — each call's copies only wait on its own kernel's
// counters).  The two events are created per call and released once enqueued (re-entrancy).
struct HostIoStreams {
    cudaStream_t copy = nullptr;  // device→host y chunks (waits on the kernel's counters)
    cudaStream_t state = nullptr; // device→host h_n / c_n per layer (waits on the kernel's counters)
    cudaStream_t h2d = nullptr;   // host→device x chunks (never waits on a kernel: no cycle
                                  // between concurrent calls sharing the streams)
    cudaEvent_t reset = nullptr, done = nullptr, xdone = nullptr, sdone = nullptr;
};
typedef CUresult (*StreamWaitValue32Fn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
typedef CUresult (*StreamWriteValue32Fn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);

bool hostio_streams(HostIoStreams* out, StreamWaitValue32Fn* wait_fn, StreamWriteValue32Fn* write_fn) {
    static HostIoStreams per_dev[64];
    static StreamWaitValue32Fn fn = nullptr;
    static StreamWriteValue32Fn wfn = nullptr;
    static std::mutex mu;
    std::lock_guard<std::mutex> lock(mu);
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return false;
    if (!fn || !wfn) {
        void* ptr = nullptr;
        void* wptr = nullptr;
        cudaDriverEntryPointQueryResult q = cudaDriverEntryPointSymbolNotFound, wq = q;
        if (cudaGetDriverEntryPointByVersion("cuStreamWaitValue32", &ptr, 12000, cudaEnableDefault, &q) !=
                cudaSuccess || q != cudaDriverEntryPointSuccess || !ptr ||
            cudaGetDriverEntryPointByVersion("cuStreamWriteValue32", &wptr, 12000, cudaEnableDefault, &wq) !=
                cudaSuccess || wq != cudaDriverEntryPointSuccess || !wptr) {
            cudaGetLastError();
            return false;
        }
        fn = reinterpret_cast<StreamWaitValue32Fn>(ptr);
        wfn = reinterpret_cast<StreamWriteValue32Fn>(wptr);
    }
    HostIoStreams& h = per_dev[dev];
    if (!h.copy && (cudaStreamCreateWithFlags(&h.copy, cudaStreamNonBlocking) != cudaSuccess ||
                    cudaStreamCreateWithFlags(&h.h2d, cudaStreamNonBlocking) != cudaSuccess ||
                    cudaStreamCreateWithFlags(&h.state, cudaStreamNonBlocking) != cudaSuccess)) {
        cudaGetLastError();
        h.copy = h.h2d = h.state = nullptr;
        return false;
    }
    *out = h;
    if (cudaEventCreateWithFlags(&out->reset, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&out->done, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&out->xdone, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&out->sdone, cudaEventDisableTiming) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    *write_fn = wfn;
    *wait_fn = fn;
    return true;
}
}  // namespace

FT_API size_t ft_stacked_lstm_hostio_workspace_size(int batch, int seq, int hidden, int depth,
                                                    ft_dtype dt) {
    const size_t inner = ft_stacked_lstm_workspace_size(batch, seq, hidden, depth, dt, 0);
    if (inner == 0) return 0;
    return plan_hostio(batch, seq, hidden, depth, dt, inner).total;
}

FT_API ft_status ft_stacked_lstm_fwd_hostio(int batch, int seq, int hidden, int depth, ft_dtype dt,
                                            const void* x_host, const void* W, const void* U,
                                            const float* b, void* y_host, void* h_n_host,
                                            float* c_n_host, void* workspace,
                                            size_t workspace_bytes, void* stream) {
    if (depth <= 0) return fail(FT_ERR_INVALID_ARGUMENT, "every dimension must be > 0");
    if (depth > FT_MAX_DEPTH) return fail(FT_ERR_UNSUPPORTED, "depth > FT_MAX_DEPTH");
    int ones[FT_MAX_DEPTH];
    for (int d = 0; d < depth; ++d) ones[d] = 1;
    ft::Problem p;
    ft_status st = make_problem(ft::KIND_SEQ, batch, seq, 1, hidden, depth, ones, dt, &p);
    if (st != FT_OK) return st;
    if (!x_host || !y_host || !h_n_host || !c_n_host)
        return fail(FT_ERR_INVALID_ARGUMENT, "a host buffer is NULL");
    REQUIRE_PTR(W, "W");
    REQUIRE_PTR(U, "U");
    REQUIRE_PTR(b, "b");
    const size_t inner = ft_stacked_lstm_workspace_size(batch, seq, hidden, depth, dt, 0);
    const HostIoPlan hp = plan_hostio(batch, seq, hidden, depth, dt, inner);
    if (!workspace) return fail(FT_ERR_INVALID_ARGUMENT, "workspace is NULL");
    if (!aligned16(workspace)) return fail(FT_ERR_INVALID_ARGUMENT, "workspace not 16-byte aligned");
    if (workspace_bytes < hp.total)
        return fail(FT_ERR_WORKSPACE_TOO_SMALL, "workspace_bytes " + std::to_string(workspace_bytes) +
                                                    " < required " + std::to_string(hp.total));
    st = check_device();
    if (st != FT_OK) return st;
    uint8_t* ws = static_cast<uint8_t*>(workspace);
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const size_t es = elem_size(dt);
    const size_t xb = (size_t)batch * seq * hidden * es, hb = (size_t)batch * depth * hidden * es;
    const size_t cb = (size_t)batch * depth * hidden * 4;
    cudaError_t e = cudaSuccess;
    ft::Tensors t;
    t.x = ws + hp.x_off;
    t.W = W;
    t.U = U;
    t.b = b;
    t.y = ws + hp.y_off;
    t.h_n = ws + hp.hn_off;
    t.c_n = reinterpret_cast<float*>(ws + hp.cn_off);
    // y leaves the device in time chunks while the nest still runs (the top layer finishes its
    // steps in order): the kernel counts each chunk's stored-and-fenced y tiles in ysig, a copy
    // stream waits for each count (cuStreamWaitValue32) and copies that chunk, and `s` waits for
    // the copy stream at the end — so the call stays stream-ordered on `s`.  Kernels that do
    // not signal (fp32, SMEM-resident, cluster) leave ysig_per_step at 0: y is copied after.
    // x likewise enters in time chunks on a second copy stream, each followed by a flag write
    // (cuStreamWriteValue32) that the streaming kernel's activation producer waits for before
    // the chunk's first layer-0 load; the kernel then reads x [B][T][H] directly (no pack).
    HostIoStreams hs;
    StreamWaitValue32Fn wait_value = nullptr;
    StreamWriteValue32Fn write_value = nullptr;
    int per_step = 0, per_chunk = 0, per_step0 = 0;
    const int chunk = hostio_chunk(), nchunks = (seq + chunk - 1) / chunk;
    const bool overlap = dt == FT_BF16 && !getenv("FT_HOSTIO_SERIAL") &&
                         ft::bf16_kernel_choice(p) == 2 && hostio_streams(&hs, &wait_value, &write_value);
    if (overlap) {
        t.ysig = reinterpret_cast<int*>(ws + hp.ysig_off);
        t.ychunk = chunk;
        t.ysig_per_step = &per_step;
        t.ysig_per_chunk = &per_chunk;
        t.nsig0_per_step = &per_step0;
        t.xsig = reinterpret_cast<int*>(ws + hp.xsig_off);
        t.xchunk = chunk;
        t.nsig = reinterpret_cast<int*>(ws + hp.nsig_off);
        e = cudaMemsetAsync(t.ysig, 0, (size_t)(hp.nsig_off - hp.ysig_off) + (size_t)depth * sizeof(int), s);
        if (e == cudaSuccess) e = cudaEventRecord(hs.reset, s);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(hs.h2d, hs.reset, 0);
        const size_t row = (size_t)seq * hidden * es;
        for (int c = 0; c < nchunks && e == cudaSuccess; ++c) {
            const int t0 = c * chunk, t1 = std::min(seq, t0 + chunk);
            const size_t off = (size_t)t0 * hidden * es;
            e = cudaMemcpy2DAsync(ws + hp.x_off + off, row, static_cast<const uint8_t*>(x_host) + off, row,
                                  (size_t)(t1 - t0) * hidden * es, batch, cudaMemcpyHostToDevice, hs.h2d);
            if (e == cudaSuccess &&
                write_value(hs.h2d, (CUdeviceptr)(t.xsig + c), 1, CU_STREAM_WRITE_VALUE_DEFAULT) != CUDA_SUCCESS)
                e = cudaErrorUnknown;
        }
        if (e == cudaSuccess) e = cudaEventRecord(hs.xdone, hs.h2d);
        if (e != cudaSuccess) {
            cudaEventDestroy(hs.reset);
            cudaEventDestroy(hs.done);
            cudaEventDestroy(hs.xdone);
            cudaEventDestroy(hs.sdone);
            return fail(FT_ERR_CUDA, std::string("hostio setup: ") + cudaGetErrorString(e));
        }
    } else {
        e = cudaMemcpyAsync(ws + hp.x_off, x_host, xb, cudaMemcpyHostToDevice, s);
        if (e != cudaSuccess) return fail(FT_ERR_CUDA, std::string("x H2D: ") + cudaGetErrorString(e));
    }
    st = run(p, dt, t, ws + hp.inner_off, inner, stream);
    if (st != FT_OK) {
        if (overlap) {  // x copies are already enqueued; keep `s` ordered after them
            cudaStreamWaitEvent(s, hs.xdone, 0);
            cudaEventDestroy(hs.reset);
            cudaEventDestroy(hs.done);
            cudaEventDestroy(hs.xdone);
            cudaEventDestroy(hs.sdone);
        }
        return st;
    }
    // h_n / c_n per layer as soon as the layer's last step is stored (nsig counters): layers of
    // earlier bands leave the device while the later bands still run
    bool state_overlapped = false;
    if (per_step > 0) {
        cudaError_t se = cudaStreamWaitEvent(hs.state, hs.reset, 0);
        const size_t hrow = (size_t)hidden * es, crow = (size_t)hidden * 4;
        const size_t hpitch = (size_t)depth * hrow, cpitch = (size_t)depth * crow;
        for (int d = 0; d < depth && se == cudaSuccess; ++d) {
            const int need = (d == 0 && per_step0 > 0) ? per_step0 : per_step;
            if (wait_value(hs.state, (CUdeviceptr)(t.nsig + d), (cuuint32_t)need, CU_STREAM_WAIT_VALUE_GEQ) !=
                CUDA_SUCCESS) {
                se = cudaErrorUnknown;
                break;
            }
            se = cudaMemcpy2DAsync(static_cast<uint8_t*>(h_n_host) + d * hrow, hpitch, ws + hp.hn_off + d * hrow,
                                   hpitch, hrow, batch, cudaMemcpyDeviceToHost, hs.state);
            if (se == cudaSuccess)
                se = cudaMemcpy2DAsync(reinterpret_cast<uint8_t*>(c_n_host) + d * crow, cpitch,
                                       ws + hp.cn_off + d * crow, cpitch, crow, batch, cudaMemcpyDeviceToHost,
                                       hs.state);
        }
        state_overlapped = se == cudaSuccess;
        if (!state_overlapped) cudaGetLastError();  // fall back below: copy after the kernel on `s`
        // `s` waits for whatever the state stream enqueued (also on the fallback path)
        if (cudaEventRecord(hs.sdone, hs.state) == cudaSuccess) cudaStreamWaitEvent(s, hs.sdone, 0);
        else state_overlapped = false;
    }
    if (per_step > 0) {
        e = cudaStreamWaitEvent(hs.copy, hs.reset, 0);
        const size_t row = (size_t)seq * hidden * es;  // one batch row of y
        for (int c = 0; c < nchunks && e == cudaSuccess; ++c) {
            const int t0 = c * chunk, t1 = std::min(seq, t0 + chunk);
            CUresult r = wait_value(hs.copy, (CUdeviceptr)(t.ysig + c),
                                    (cuuint32_t)((per_chunk ? 1 : t1 - t0) * per_step), CU_STREAM_WAIT_VALUE_GEQ);
            if (r != CUDA_SUCCESS) {  // fall back: copy the rest of y on `s` after the kernel
                e = cudaMemcpy2DAsync(static_cast<uint8_t*>(y_host) + (size_t)t0 * hidden * es, row,
                                      ws + hp.y_off + (size_t)t0 * hidden * es, row,
                                      (size_t)(seq - t0) * hidden * es, batch, cudaMemcpyDeviceToHost, s);
                break;
            }
            const size_t off = (size_t)t0 * hidden * es;
            e = cudaMemcpy2DAsync(static_cast<uint8_t*>(y_host) + off, row, ws + hp.y_off + off, row,
                                  (size_t)(t1 - t0) * hidden * es, batch, cudaMemcpyDeviceToHost, hs.copy);
        }
        if (e == cudaSuccess) e = cudaEventRecord(hs.done, hs.copy);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(s, hs.done, 0);
    } else {
        e = cudaMemcpyAsync(y_host, ws + hp.y_off, xb, cudaMemcpyDeviceToHost, s);
    }
    if (overlap) {  // destroying an enqueued event is safe: released when it completes
        if (e == cudaSuccess) e = cudaStreamWaitEvent(s, hs.xdone, 0);
        cudaEventDestroy(hs.reset);
        cudaEventDestroy(hs.done);
        cudaEventDestroy(hs.xdone);
        cudaEventDestroy(hs.sdone);
    }
    if (!state_overlapped) {
        if (e == cudaSuccess) e = cudaMemcpyAsync(h_n_host, ws + hp.hn_off, hb, cudaMemcpyDeviceToHost, s);
        if (e == cudaSuccess) e = cudaMemcpyAsync(c_n_host, ws + hp.cn_off, cb, cudaMemcpyDeviceToHost, s);
    }
    if (e != cudaSuccess) return fail(FT_ERR_CUDA, std::string("D2H: ") + cudaGetErrorString(e));
    return FT_OK;
}

FT_API size_t ft_stacked_lstm_layerwise_workspace_size(int batch, int seq, int hidden, int depth,
                                                       ft_dtype dt) {
    if (dt != FT_BF16 || depth <= 0 || depth > FT_MAX_DEPTH || batch <= 0 || seq <= 0 || hidden <= 0 ||
        hidden % 64 != 0)
        return 0;
    return ft::layerwise_ws_bytes(batch, seq, hidden);
}

FT_API ft_status ft_stacked_lstm_layerwise_fwd(int batch, int seq, int hidden, int depth, ft_dtype dt,
                                               const void* x, const void* W, const void* U,
                                               const float* b, void* y, void* h_n, float* c_n,
                                               void* h_all, float* c_all, void* workspace,
                                               size_t workspace_bytes, void* stream) {
    if (dt != FT_F32 && dt != FT_BF16) return fail(FT_ERR_INVALID_ARGUMENT, "unknown dtype");
    if (batch <= 0 || seq <= 0 || hidden <= 0 || depth <= 0)
        return fail(FT_ERR_INVALID_ARGUMENT, "every dimension must be > 0");
    if (depth > FT_MAX_DEPTH) return fail(FT_ERR_UNSUPPORTED, "depth > FT_MAX_DEPTH");
    if (dt != FT_BF16) return fail(FT_ERR_UNSUPPORTED, "the layer-sequential schedule is bf16 only");
    if (hidden % 64 != 0) return fail(FT_ERR_UNSUPPORTED, "bf16 path requires hidden % 64 == 0");
    if ((long long)batch * seq * 4 * hidden >= (1ll << 31) ||
        (long long)seq * hidden * ((batch + 127) / 128 * 128) / 64 >= (1ll << 31))
        return fail(FT_ERR_UNSUPPORTED, "problem too large for 32-bit GEMM / TMA coordinates");
    REQUIRE_PTR(x, "x");
    REQUIRE_PTR(W, "W");
    REQUIRE_PTR(U, "U");
    REQUIRE_PTR(b, "b");
    REQUIRE_PTR(y, "y");
    REQUIRE_PTR(h_n, "h_n");
    REQUIRE_PTR(c_n, "c_n");
    OPTIONAL_PTR(h_all, "h_all");
    OPTIONAL_PTR(c_all, "c_all");
    const size_t need = ft::layerwise_ws_bytes(batch, seq, hidden);
    if (!workspace) return fail(FT_ERR_INVALID_ARGUMENT, "workspace is NULL");
    if (!aligned16(workspace)) return fail(FT_ERR_INVALID_ARGUMENT, "workspace not 16-byte aligned");
    if (workspace_bytes < need)
        return fail(FT_ERR_WORKSPACE_TOO_SMALL, "workspace_bytes " + std::to_string(workspace_bytes) +
                                                    " < required " + std::to_string(need));
    ft_status st = check_device();
    if (st != FT_OK) return st;
    int dev = 0, nsm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    std::string why;
    if (ft::layerwise_supported(batch, hidden, nsm, &why) != 0) return fail(FT_ERR_UNSUPPORTED, why);
    std::string err;
    PersistentOrder order(static_cast<cudaStream_t>(stream));
    cudaError_t e = ft::launch_layerwise(batch, seq, hidden, depth, x, W, U, b, y, h_n, c_n, h_all,
                                         c_all, workspace, static_cast<cudaStream_t>(stream), &err);
    if (e != cudaSuccess) return fail(FT_ERR_CUDA, err.empty() ? cudaGetErrorString(e) : err);
    return FT_OK;
}

FT_API size_t ft_stacked_rnn_workspace_size(int batch, int seq, int hidden, int depth, ft_dtype dt) {
    if (depth <= 0 || depth > FT_MAX_DEPTH) return 0;
    int ones[FT_MAX_DEPTH];
    for (int d = 0; d < depth; ++d) ones[d] = 1;
    ft::Problem p;
    if (make_problem(ft::KIND_SEQ, batch, seq, 1, hidden, depth, ones, dt, &p, ft::CELL_LINEAR) != FT_OK)
        return 0;
    return plan_workspace(p, dt, true).total;
}

FT_API ft_status ft_stacked_rnn_fwd(int batch, int seq, int hidden, int depth, ft_dtype dt,
                                    const void* x, const void* W, void* ys, void* workspace,
                                    size_t workspace_bytes, void* stream) {
    if (depth <= 0) return fail(FT_ERR_INVALID_ARGUMENT, "every dimension must be > 0");
    if (depth > FT_MAX_DEPTH) return fail(FT_ERR_UNSUPPORTED, "depth > FT_MAX_DEPTH");
    int ones[FT_MAX_DEPTH];
    for (int d = 0; d < depth; ++d) ones[d] = 1;
    ft::Problem p;
    ft_status st = make_problem(ft::KIND_SEQ, batch, seq, 1, hidden, depth, ones, dt, &p, ft::CELL_LINEAR);
    if (st != FT_OK) return st;
    REQUIRE_PTR(x, "x");
    REQUIRE_PTR(W, "W");
    REQUIRE_PTR(ys, "ys");
    ft::Tensors t;
    t.x = x;
    t.W = W;
    t.h_all = ys;  // Listing 1's ysss [N, D, L] is the SSA buffer itself
    return run(p, dt, t, workspace, workspace_bytes, stream);
}

FT_API size_t ft_dilated_rnn_workspace_size(int batch, int seq, int hidden, int depth,
                                            const int* dilations, ft_dtype dt, int h_all_provided) {
    ft::Problem p;
    if (make_problem(ft::KIND_SEQ, batch, seq, 1, hidden, depth, dilations, dt, &p) != FT_OK) return 0;
    return plan_workspace(p, dt, h_all_provided != 0).total;
}

FT_API ft_status ft_dilated_rnn_fwd(int batch, int seq, int hidden, int depth, const int* dilations,
                                    ft_dtype dt, const void* x, const void* W, const void* U,
                                    const float* b, void* y, void* h_n, float* c_n, void* h_all,
                                    float* c_all, void* workspace, size_t workspace_bytes,
                                    void* stream) {
    return seq_fwd(batch, seq, hidden, depth, dilations, dt, x, W, U, b, y, h_n, c_n, h_all, c_all,
                   workspace, workspace_bytes, stream);
}

FT_API size_t ft_grid_rnn_workspace_size(int batch, int len_x, int len_y, int hidden, int depth,
                                         ft_dtype dt, int h_all_provided) {
    ft::Problem p;
    if (make_problem(ft::KIND_GRID, batch, len_x, len_y, hidden, depth, nullptr, dt, &p) != FT_OK)
        return 0;
    return plan_workspace(p, dt, h_all_provided != 0).total;
}

FT_API ft_status ft_grid_rnn_fwd(int batch, int len_x, int len_y, int hidden, int depth, ft_dtype dt,
                                 const void* x, const void* ys, const void* W, const void* U,
                                 const float* b, void* out, void* h_n, float* c_n, void* h_all,
                                 float* c_all, void* workspace, size_t workspace_bytes,
                                 void* stream) {
    ft::Problem p;
    ft_status st = make_problem(ft::KIND_GRID, batch, len_x, len_y, hidden, depth, nullptr, dt, &p);
    if (st != FT_OK) return st;
    REQUIRE_PTR(x, "x");
    REQUIRE_PTR(ys, "ys");
    REQUIRE_PTR(W, "W");
    REQUIRE_PTR(U, "U");
    REQUIRE_PTR(b, "b");
    REQUIRE_PTR(out, "out");
    REQUIRE_PTR(h_n, "h_n");
    REQUIRE_PTR(c_n, "c_n");
    OPTIONAL_PTR(h_all, "h_all");
    OPTIONAL_PTR(c_all, "c_all");
    ft::Tensors t;
    t.x = x;
    t.ys = ys;
    t.W = W;
    t.U = U;
    t.b = b;
    t.y = out;
    t.h_n = h_n;
    t.c_n = c_n;
    t.h_all = h_all;
    t.c_all = c_all;
    return run(p, dt, t, workspace, workspace_bytes, stream);
}

FT_API long long ft_wavefront_cells(int kind, int depth, int len_a, int len_b, int* out_cells,
                                    long long cap) {
    return ft_wavefront_cells_banded(kind, depth, len_a, len_b, 0, 1, out_cells, cap);
}

FT_API long long ft_wavefront_cells_banded(int kind, int depth, int len_a, int len_b, int band,
                                           int skew, int* out_cells, long long cap) {
    if (kind != ft::KIND_SEQ && kind != ft::KIND_GRID) return -1;
    if (kind == ft::KIND_SEQ) len_b = 1;
    if (depth <= 0 || len_a <= 0 || len_b <= 0 || depth > FT_MAX_DEPTH) return -1;
    if (cap > 0 && !out_cells) return -1;
    ft::Problem p;
    std::memset(&p, 0, sizeof(p));
    p.kind = kind;
    p.D = depth;
    p.L0 = len_a;
    p.L1 = len_b;
    p.B = p.H = 1;
    p.naxes = kind == ft::KIND_SEQ ? 1 : 2;
    p.MB = p.NT = 1;
    p.ncells = (long long)depth * len_a * len_b;
    p.band = band;
    p.skew = kind == ft::KIND_SEQ ? skew : 1;
    ft::Cursor cur = ft::cursor_begin();
    for (long long o = 0; o < p.ncells; ++o) {
        ft::cursor_seek(p, cur, o);
        if (o < cap) {
            out_cells[4 * o + 0] = cur.cell.k;
            out_cells[4 * o + 1] = cur.cell.d;
            out_cells[4 * o + 2] = cur.cell.i;
            out_cells[4 * o + 3] = cur.cell.j;
        }
    }
    return p.ncells;
}

FT_API long long ft_tile_walk(int depth, int seq, int band, int skew, int owner, int ntiles_n,
                              int worker, int nworkers, int* out, long long cap) {
    if (depth <= 0 || seq <= 0 || depth > FT_MAX_DEPTH || ntiles_n <= 0 || nworkers <= 0 ||
        worker < 0 || worker >= nworkers || (cap > 0 && !out))
        return -1;
    ft::Problem p;
    std::memset(&p, 0, sizeof(p));
    p.kind = ft::KIND_SEQ;
    p.D = depth;
    p.L0 = seq;
    p.L1 = 1;
    p.B = p.H = 1;
    p.naxes = 1;
    p.MB = 1;
    p.NT = ntiles_n;
    p.ncells = (long long)depth * seq;
    p.ntiles = p.ncells * ntiles_n;
    p.band = band;
    p.skew = skew;
    p.owner = (owner == 1 && band > 0 && band < depth && ft::seq_band(p) * ntiles_n <= nworkers)
                  ? 1
                  : (owner == 2 && 2 * ntiles_n <= nworkers ? 2
                     : (owner == 3 && depth * ntiles_n <= nworkers ? 3
                     : (owner == 4 && (depth + 1) * ntiles_n <= nworkers ? 3 : 0)));
    if (owner == 4 && p.owner == 3) p.nt0 = 2 * ntiles_n;
    for (int d = 0; d < depth; ++d) p.dil[d] = 1;
    ft::TileWalk w = ft::walk_begin(p, worker, nworkers);
    ft::TileId tl;
    long long tid = 0, n = 0;
    while (ft::walk_next(p, w, tl, tid)) {
        if (n < cap) {
            out[3 * n + 0] = tl.cell.d;
            out[3 * n + 1] = tl.cell.i;
            out[3 * n + 2] = tl.n;
        }
        ++n;
    }
    return n;
}

FT_API ft_status ft_b2b_gemm_fwd(int M, int N, int K, int P, ft_dtype dt, const void* A,
                                 const void* B, const void* C, float* D, void* stream) {
    if (dt != FT_F32 && dt != FT_BF16) return fail(FT_ERR_INVALID_ARGUMENT, "unknown dtype");
    if (M <= 0 || N <= 0 || K <= 0 || P <= 0)
        return fail(FT_ERR_INVALID_ARGUMENT, "every dimension must be > 0");
    REQUIRE_PTR(A, "A");
    REQUIRE_PTR(B, "B");
    REQUIRE_PTR(C, "C");
    REQUIRE_PTR(D, "D");
    if (dt != FT_BF16 || K != 64 || P != 64 || M % 128 != 0 || N % 128 != 0)
        return fail(FT_ERR_UNSUPPORTED,
                    "b2b GEMM supports bf16 with K = P = 64 (Table 6) and M, N multiples of 128");
    if ((long long)M * 64 >= (1ll << 31) || (long long)N >= (1ll << 30))
        return fail(FT_ERR_UNSUPPORTED, "problem too large for 32-bit coordinates");
    ft_status st = check_device();
    if (st != FT_OK) return st;
    std::string err;
    cudaError_t e = ft::launch_b2b_gemm(M, N, A, B, C, D, static_cast<cudaStream_t>(stream), &err);
    if (e != cudaSuccess) return fail(FT_ERR_CUDA, err.empty() ? cudaGetErrorString(e) : err);
    return FT_OK;
}

FT_API long long ft_ssa_slots(int depth, int seq, const int* dilations, int band, int* off, int* mask) {
    if (depth <= 0 || seq <= 0 || depth > FT_MAX_DEPTH || !dilations || !off || !mask) return -1;
    ft::Problem p;
    std::memset(&p, 0, sizeof(p));
    p.kind = ft::KIND_SEQ;
    p.D = depth;
    p.L0 = seq;
    p.L1 = 1;
    long long rows = 2ll * seq;
    for (int d = 0; d < depth; ++d) {
        if (dilations[d] < 1) return -1;
        p.dil[d] = dilations[d];
        rows += ft::hb_ring_len(dilations[d], seq);
    }
    ft::hb_layout(p, band > 0 && band < depth ? band : 0);
    for (int d = 0; d < depth; ++d) {
        off[d] = p.hb_off[d];
        mask[d] = p.hb_mask[d];
    }
    return rows;
}
