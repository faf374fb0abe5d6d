// ft_comm.cu — the north star's final output gather as a C-ABI call:
// one process driving several GPUs, an NCCL communicator over them (ncclCommInitAll), and a
// gather of every device's output slice to a root device (NCCL send/recv inside one group —
// NVLink / NVSwitch on a B200 node).  The batch map is fully parallel (Table 1), so
// the gather is the only collective the path has; the forward itself exchanges nothing.
//
// NCCL is loaded at run time (libnccl.so.2: the torch-bundled or the system library), so libft.so
// has no link-time dependency on it; a missing NCCL surfaces as FT_ERR_NCCL from ft_comm_create.
// Host code only: argument checks, communicator lifetime, and the group of send/recv calls.
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
typedef int (*NcclCommDestroy)(nccl_comm_t);
typedef int (*NcclGroup)(void);
typedef int (*NcclSend)(const void*, size_t, int, int, nccl_comm_t, cudaStream_t);
typedef int (*NcclRecv)(void*, size_t, int, int, nccl_comm_t, cudaStream_t);
typedef const char* (*NcclErr)(int);
constexpr int NCCL_UINT8 = 1;

struct Nccl {
    void* lib = nullptr;
    NcclCommInitAll init_all = nullptr;
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
        if (!n.init_all || !n.destroy || !n.group_start || !n.group_end || !n.send || !n.recv) {
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

struct ft_comm {
    std::vector<int> devices;
    std::vector<nccl_comm_t> comms;
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
