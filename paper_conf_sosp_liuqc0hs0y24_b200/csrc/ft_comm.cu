// ft_comm.cu — the north star's final output gather as a C-ABI call:
// one process driving several GPUs, an NCCL communicator over them (ncclCommInitAll), and a
// gather of every device's output slice to a root device (NCCL send/recv inside one group —
// NVLink / NVSwitch on a B200 node).  The batch map is fully parallel (Table 1), so
// the gather is the only collective the path has; the forward itself exchanges nothing.
//
// NCCL is loaded at run time (libnccl.so.2: the torch-bundled or the system library), so libft.so
// has no link-time dependency on it; a missing NCCL surfaces as FT_ERR_NCCL from ft_comm_create.
// Host code only: argument checks, communicator lifetime, and the group of send/recv calls.
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstdint>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/ft.h"

#define FT_API extern "C" __attribute__((visibility("default")))

namespace {

// the subset of nccl.h this file uses (types are ABI-stable: opaque pointers and ints)
typedef void* nccl_comm_t;
typedef int (*NcclCommInitAll)(nccl_comm_t*, int, const int*);
struct NcclUniqueId { char internal[FT_COMM_ID_BYTES]; };  // ncclUniqueId (128 bytes, by value)
typedef int (*NcclGetUniqueId)(NcclUniqueId*);
typedef int (*NcclCommInitRank)(nccl_comm_t*, int, NcclUniqueId, int);
typedef int (*NcclCommDestroy)(nccl_comm_t);
typedef int (*NcclGroup)(void);
typedef int (*NcclSend)(const void*, size_t, int, int, nccl_comm_t, cudaStream_t);
typedef int (*NcclRecv)(void*, size_t, int, int, nccl_comm_t, cudaStream_t);
typedef const char* (*NcclErr)(int);
constexpr int NCCL_UINT8 = 1;

struct Nccl {
    void* lib = nullptr;
    NcclCommInitAll init_all = nullptr;
    NcclGetUniqueId get_id = nullptr;
    NcclCommInitRank init_rank = nullptr;
    NcclCommDestroy destroy = nullptr;
    NcclGroup group_start = nullptr, group_end = nullptr;
    NcclSend send = nullptr;
    NcclRecv recv = nullptr;
    NcclErr err = nullptr;
};

thread_local std::string g_comm_error;

Nccl* nccl() {
    static Nccl n;
    if (!n.lib) {
        for (const char* nm : {"libnccl.so.2", "libnccl.so"})
            if ((n.lib = dlopen(nm, RTLD_NOW | RTLD_GLOBAL))) break;
        if (!n.lib) return nullptr;
        n.init_all = (NcclCommInitAll)dlsym(n.lib, "ncclCommInitAll");
        n.destroy = (NcclCommDestroy)dlsym(n.lib, "ncclCommDestroy");
        n.group_start = (NcclGroup)dlsym(n.lib, "ncclGroupStart");
        n.group_end = (NcclGroup)dlsym(n.lib, "ncclGroupEnd");
        n.send = (NcclSend)dlsym(n.lib, "ncclSend");
        n.recv = (NcclRecv)dlsym(n.lib, "ncclRecv");
        n.err = (NcclErr)dlsym(n.lib, "ncclGetErrorString");
        n.get_id = (NcclGetUniqueId)dlsym(n.lib, "ncclGetUniqueId");
        n.init_rank = (NcclCommInitRank)dlsym(n.lib, "ncclCommInitRank");
        if (!n.get_id || !n.init_rank || !n.init_all || !n.destroy || !n.group_start || !n.group_end || !n.send || !n.recv) {
            n.lib = nullptr;
            return nullptr;
        }
    }
    return &n;
}

std::string nccl_msg(Nccl* n, int rc) {
    return std::string("NCCL error ") + std::to_string(rc) + (n && n->err ? std::string(": ") + n->err(rc) : "");
}

}  // namespace

// One-process form (ft_comm_create): devices.size() communicators, rank r on devices[r].
// Multi-process form (ft_comm_init_rank): one communicator, this process's `rank` of `nranks`.
struct ft_comm {
    std::vector<int> devices;
    std::vector<nccl_comm_t> comms;
    int nranks = 0, rank = -1;  // multi-process form only (rank >= 0)
};

// ft_last_error() lives in ft_api.cu; comm errors are reported through it as well.
namespace ft {
void set_last_error(const std::string& msg);
}

static ft_status comm_fail(ft_status s, const std::string& msg) {
    ft::set_last_error(msg);
    return s;
}

FT_API ft_status ft_comm_create(int ndev, const int* devices, ft_comm** out) {
    if (!out) return comm_fail(FT_ERR_INVALID_ARGUMENT, "out is NULL");
    *out = nullptr;
    if (ndev <= 0 || !devices) return comm_fail(FT_ERR_INVALID_ARGUMENT, "ndev must be > 0 and devices non-NULL");
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count <= 0)
        return comm_fail(FT_ERR_CUDA, "no usable CUDA device");
    for (int i = 0; i < ndev; ++i) {
        if (devices[i] < 0 || devices[i] >= count)
            return comm_fail(FT_ERR_INVALID_ARGUMENT, "device id out of range: " + std::to_string(devices[i]));
        for (int j = 0; j < i; ++j)
            if (devices[j] == devices[i])
                return comm_fail(FT_ERR_INVALID_ARGUMENT, "duplicate device id " + std::to_string(devices[i]));
    }
    Nccl* n = nccl();
    if (!n) return comm_fail(FT_ERR_NCCL, "libnccl.so.2 not found or incomplete");
    ft_comm* c = new ft_comm;
    c->devices.assign(devices, devices + ndev);
    c->comms.assign(ndev, nullptr);
    const int rc = n->init_all(c->comms.data(), ndev, devices);
    if (rc != 0) {
        delete c;
        return comm_fail(FT_ERR_NCCL, "ncclCommInitAll: " + nccl_msg(n, rc));
    }
    *out = c;
    return FT_OK;
}

FT_API ft_status ft_comm_gather(ft_comm* c, const void* const* send, void* recv, const size_t* bytes,
                                int root, void* const* streams) {
    if (!c) return comm_fail(FT_ERR_INVALID_ARGUMENT, "comm is NULL");
    if (c->rank >= 0) return comm_fail(FT_ERR_INVALID_ARGUMENT, "comm was made by ft_comm_init_rank: use ft_comm_gather_rank");
    const int nd = (int)c->devices.size();
    if (!send || !bytes || !streams) return comm_fail(FT_ERR_INVALID_ARGUMENT, "send/bytes/streams is NULL");
    if (root < 0 || root >= nd) return comm_fail(FT_ERR_INVALID_ARGUMENT, "root out of range");
    if (!recv) return comm_fail(FT_ERR_INVALID_ARGUMENT, "recv is NULL");
    for (int r = 0; r < nd; ++r)
        if (bytes[r] > 0 && !send[r]) return comm_fail(FT_ERR_INVALID_ARGUMENT, "send[r] is NULL");
    Nccl* n = nccl();
    if (!n) return comm_fail(FT_ERR_NCCL, "libnccl.so.2 not available");
    int prev = 0;
    cudaGetDevice(&prev);
    // root's own slice: a device-local copy on the root stream; the others arrive by NCCL.
    size_t off = 0;
    std::vector<size_t> offs(nd);
    for (int r = 0; r < nd; ++r) {
        offs[r] = off;
        off += bytes[r];
    }
    uint8_t* dst = static_cast<uint8_t*>(recv);
    if (cudaSetDevice(c->devices[root]) != cudaSuccess)
        return comm_fail(FT_ERR_CUDA, "cudaSetDevice(root) failed");
    if (bytes[root] > 0 &&
        cudaMemcpyAsync(dst + offs[root], send[root], bytes[root], cudaMemcpyDeviceToDevice,
                        static_cast<cudaStream_t>(streams[root])) != cudaSuccess) {
        cudaSetDevice(prev);
        return comm_fail(FT_ERR_CUDA, "root slice copy failed");
    }
    int rc = n->group_start();
    for (int r = 0; r < nd && rc == 0; ++r) {
        if (r == root || bytes[r] == 0) continue;
        rc = n->send(send[r], bytes[r], NCCL_UINT8, root, c->comms[r], static_cast<cudaStream_t>(streams[r]));
        if (rc == 0)
            rc = n->recv(dst + offs[r], bytes[r], NCCL_UINT8, r, c->comms[root],
                         static_cast<cudaStream_t>(streams[root]));
    }
    const int rc2 = n->group_end();
    cudaSetDevice(prev);
    if (rc != 0 || rc2 != 0) return comm_fail(FT_ERR_NCCL, "gather: " + nccl_msg(n, rc ? rc : rc2));
    return FT_OK;
}

FT_API ft_status ft_comm_destroy(ft_comm* c) {
    if (!c) return FT_OK;
    Nccl* n = nccl();
    int rc = 0;
    for (nccl_comm_t cm : c->comms)
        if (cm && n) rc |= n->destroy(cm);
    delete c;
    if (rc != 0) return comm_fail(FT_ERR_NCCL, "ncclCommDestroy failed");
    return FT_OK;
}

// ------------------------------------------------------------------------------ one process per GPU
FT_API ft_status ft_comm_unique_id(void* id) {
    if (!id) return comm_fail(FT_ERR_INVALID_ARGUMENT, "id is NULL");
    Nccl* n = nccl();
    if (!n) return comm_fail(FT_ERR_NCCL, "libnccl.so.2 not found or incomplete");
    NcclUniqueId u;
    const int rc = n->get_id(&u);
    if (rc != 0) return comm_fail(FT_ERR_NCCL, "ncclGetUniqueId: " + nccl_msg(n, rc));
    std::memcpy(id, u.internal, FT_COMM_ID_BYTES);
    return FT_OK;
}

FT_API ft_status ft_comm_init_rank(int nranks, int rank, const void* id, int device, ft_comm** out) {
    if (!out) return comm_fail(FT_ERR_INVALID_ARGUMENT, "out is NULL");
    *out = nullptr;
    if (nranks <= 0 || rank < 0 || rank >= nranks || !id)
        return comm_fail(FT_ERR_INVALID_ARGUMENT, "need 0 <= rank < nranks and a non-NULL id");
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count <= 0)
        return comm_fail(FT_ERR_CUDA, "no usable CUDA device");
    if (device < 0 || device >= count)
        return comm_fail(FT_ERR_INVALID_ARGUMENT, "device id out of range: " + std::to_string(device));
    Nccl* n = nccl();
    if (!n) return comm_fail(FT_ERR_NCCL, "libnccl.so.2 not found or incomplete");
    int prev = 0;
    cudaGetDevice(&prev);
    if (cudaSetDevice(device) != cudaSuccess) return comm_fail(FT_ERR_CUDA, "cudaSetDevice failed");
    NcclUniqueId u;
    std::memcpy(u.internal, id, FT_COMM_ID_BYTES);
    nccl_comm_t cm = nullptr;
    const int rc = n->init_rank(&cm, nranks, u, rank);
    cudaSetDevice(prev);
    if (rc != 0) return comm_fail(FT_ERR_NCCL, "ncclCommInitRank: " + nccl_msg(n, rc));
    ft_comm* c = new ft_comm;
    c->devices.assign(1, device);
    c->comms.assign(1, cm);
    c->nranks = nranks;
    c->rank = rank;
    *out = c;
    return FT_OK;
}

FT_API ft_status ft_comm_gather_rank(ft_comm* c, const void* send, void* recv, const size_t* bytes,
                                     int root, void* stream) {
    if (!c) return comm_fail(FT_ERR_INVALID_ARGUMENT, "comm is NULL");
    if (c->rank < 0) return comm_fail(FT_ERR_INVALID_ARGUMENT, "comm was not made by ft_comm_init_rank");
    const int nr = c->nranks;
    if (!bytes) return comm_fail(FT_ERR_INVALID_ARGUMENT, "bytes is NULL");
    if (root < 0 || root >= nr) return comm_fail(FT_ERR_INVALID_ARGUMENT, "root out of range");
    if (bytes[c->rank] > 0 && !send) return comm_fail(FT_ERR_INVALID_ARGUMENT, "send is NULL");
    if (c->rank == root && !recv) return comm_fail(FT_ERR_INVALID_ARGUMENT, "recv is NULL on the root");
    Nccl* n = nccl();
    if (!n) return comm_fail(FT_ERR_NCCL, "libnccl.so.2 not available");
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    int prev = 0;
    cudaGetDevice(&prev);
    if (cudaSetDevice(c->devices[0]) != cudaSuccess) return comm_fail(FT_ERR_CUDA, "cudaSetDevice failed");
    int rc = 0;
    if (c->rank == root) {
        uint8_t* dst = static_cast<uint8_t*>(recv);
        size_t off = 0, own = 0;
        for (int r = 0; r < root; ++r) own += bytes[r];
        // the root's own slice: in place when the caller computed it there (send == recv + own)
        if (bytes[root] > 0 && send != dst + own &&
            cudaMemcpyAsync(dst + own, send, bytes[root], cudaMemcpyDeviceToDevice, s) != cudaSuccess) {
            cudaSetDevice(prev);
            return comm_fail(FT_ERR_CUDA, "root slice copy failed");
        }
        rc = n->group_start();
        for (int r = 0; r < nr && rc == 0; ++r) {
            if (r != root && bytes[r] > 0) rc = n->recv(dst + off, bytes[r], NCCL_UINT8, r, c->comms[0], s);
            off += bytes[r];
        }
        const int rc2 = n->group_end();
        if (rc == 0) rc = rc2;
    } else if (bytes[c->rank] > 0) {
        rc = n->send(send, bytes[c->rank], NCCL_UINT8, root, c->comms[0], s);
    }
    cudaSetDevice(prev);
    if (rc != 0) return comm_fail(FT_ERR_NCCL, "gather: " + nccl_msg(n, rc));
    return FT_OK;
}

// ------------------------------------------------------------------------------ peer memory
// NEXT-1's fused gather: rank `dst` exports its output buffers, every other rank maps them into
// its own device's address space (CUDA IPC; on an NVSwitch node a peer-to-peer NVLink window) and
// hands its row slice to the forward as y / h_n / c_n, so the kernel epilogue's stores are the
// gather.  Host plumbing only.
namespace {
typedef CUresult (*MemGetAddressRangeFn)(CUdeviceptr*, size_t*, CUdeviceptr);
MemGetAddressRangeFn addr_range_fn() {
    static MemGetAddressRangeFn fn = nullptr;
    if (!fn) {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q = cudaDriverEntryPointSymbolNotFound;
        if (cudaGetDriverEntryPointByVersion("cuMemGetAddressRange", &p, 12000, cudaEnableDefault, &q) ==
                cudaSuccess && q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<MemGetAddressRangeFn>(p);
    }
    return fn;
}
}  // namespace

FT_API ft_status ft_ipc_export(const void* dev_ptr, void* handle, size_t* offset) {
    if (!dev_ptr || !handle || !offset) return comm_fail(FT_ERR_INVALID_ARGUMENT, "NULL argument");
    static_assert(sizeof(cudaIpcMemHandle_t) == FT_IPC_HANDLE_BYTES, "IPC handle size");
    MemGetAddressRangeFn range = addr_range_fn();
    if (!range) return comm_fail(FT_ERR_CUDA, "cuMemGetAddressRange not available from the driver");
    CUdeviceptr base = 0;
    size_t size = 0;
    if (range(&base, &size, reinterpret_cast<CUdeviceptr>(dev_ptr)) != CUDA_SUCCESS)
        return comm_fail(FT_ERR_INVALID_ARGUMENT, "not a device allocation");
    cudaIpcMemHandle_t h;
    const cudaError_t e = cudaIpcGetMemHandle(&h, reinterpret_cast<void*>(base));
    if (e != cudaSuccess) {
        cudaGetLastError();
        return comm_fail(FT_ERR_CUDA, std::string("cudaIpcGetMemHandle: ") + cudaGetErrorString(e));
    }
    std::memcpy(handle, &h, FT_IPC_HANDLE_BYTES);
    *offset = reinterpret_cast<uintptr_t>(dev_ptr) - (uintptr_t)base;
    return FT_OK;
}

FT_API ft_status ft_ipc_open(const void* handle, size_t offset, int device, void** dev_ptr) {
    if (!handle || !dev_ptr) return comm_fail(FT_ERR_INVALID_ARGUMENT, "NULL argument");
    *dev_ptr = nullptr;
    int prev = 0;
    cudaGetDevice(&prev);
    if (cudaSetDevice(device) != cudaSuccess) {
        cudaGetLastError();
        return comm_fail(FT_ERR_INVALID_ARGUMENT, "bad device id");
    }
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle, FT_IPC_HANDLE_BYTES);
    void* base = nullptr;
    const cudaError_t e = cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess);
    cudaSetDevice(prev);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return comm_fail(FT_ERR_CUDA, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
    }
    *dev_ptr = static_cast<uint8_t*>(base) + offset;
    return FT_OK;
}

FT_API ft_status ft_ipc_close(void* dev_ptr, size_t offset) {
    if (!dev_ptr) return FT_OK;
    const cudaError_t e = cudaIpcCloseMemHandle(static_cast<uint8_t*>(dev_ptr) - offset);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return comm_fail(FT_ERR_CUDA, std::string("cudaIpcCloseMemHandle: ") + cudaGetErrorString(e));
    }
    return FT_OK;
}
