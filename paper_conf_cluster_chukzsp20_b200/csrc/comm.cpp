// comm.cpp -- NCCL (resolved at run time from the copy torch already loaded)
// and CUDA-IPC device windows: the plumbing under ddt_exchange.
//
// NCCL is bound lazily with dlopen/dlsym so that the library loads (and the
// CPU test-suite runs) without NCCL present; on a GPU box `import torch`
// has already mapped torch's libnccl.so.2 (2.28.9), and RTLD_NOLOAD picks up
// that very copy, so communicators created here and torch's agree on the ABI.
#include <dlfcn.h>

#include <cstring>
#include <mutex>
#include <string>

#include <cuda_runtime.h>

#include "ddt_internal.h"
#include "nccl_min.h"

namespace ddt {

static NcclApi g_nccl;
static std::once_flag g_nccl_once;

static void load_nccl() {
    const char* names[] = {"libnccl.so.2", "libnccl.so"};
    void* h = nullptr;
    for (const char* n : names) {
        h = dlopen(n, RTLD_NOW | RTLD_NOLOAD | RTLD_GLOBAL);
        if (h) break;
    }
    if (!h) {
        const char* env = getenv("DDT_NCCL_LIB");
        if (env) h = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
    }
    if (!h) {
        for (const char* n : names) {
            h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
            if (h) break;
        }
    }
    if (!h) return;
#define DDT_SYM(field, name) g_nccl.field = (decltype(g_nccl.field))dlsym(h, name)
    DDT_SYM(GetUniqueId, "ncclGetUniqueId");
    DDT_SYM(CommInitRank, "ncclCommInitRank");
    DDT_SYM(CommDestroy, "ncclCommDestroy");
    DDT_SYM(Send, "ncclSend");
    DDT_SYM(Recv, "ncclRecv");
    DDT_SYM(AllReduce, "ncclAllReduce");
    DDT_SYM(GroupStart, "ncclGroupStart");
    DDT_SYM(GroupEnd, "ncclGroupEnd");
    DDT_SYM(GetErrorString, "ncclGetErrorString");
    DDT_SYM(CommGetAsyncError, "ncclCommGetAsyncError");
#undef DDT_SYM
    g_nccl.ok = g_nccl.GetUniqueId && g_nccl.CommInitRank && g_nccl.Send && g_nccl.Recv && g_nccl.GroupStart &&
                g_nccl.GroupEnd && g_nccl.CommDestroy && g_nccl.AllReduce;
}

const NcclApi* nccl() {
    std::call_once(g_nccl_once, load_nccl);
    return g_nccl.ok ? &g_nccl : nullptr;
}

ddt_status_t alloc_base(const void* p, void** base) {
    using GetRange = int (*)(unsigned long long*, size_t*, unsigned long long);
    static GetRange fn = [] {
        void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_NOLOAD);
        if (!h) h = dlopen("libcuda.so.1", RTLD_NOW);
        return h ? (GetRange)dlsym(h, "cuMemGetAddressRange_v2") : (GetRange) nullptr;
    }();
    if (!fn) {
        set_error("cuMemGetAddressRange unavailable");
        return DDT_ERR_UNSUPPORTED;
    }
    unsigned long long b = 0;
    size_t sz = 0;
    int r = fn(&b, &sz, (unsigned long long)(uintptr_t)p);
    if (r != 0) {
        set_error("cuMemGetAddressRange failed (" + std::to_string(r) + ")");
        return DDT_ERR_CUDA;
    }
    *base = (void*)(uintptr_t)b;
    return DDT_OK;
}

ddt_status_t nccl_fail(const char* what, int r) {
    const NcclApi* n = nccl();
    std::string m = std::string(what) + ": nccl error " + std::to_string(r);
    if (n && n->GetErrorString) m += std::string(" (") + n->GetErrorString(r) + ")";
    set_error(m);
    return DDT_ERR_NCCL;
}

}  // namespace ddt

using namespace ddt;

extern "C" {

ddt_status_t ddt_nccl_unique_id(void* id_out) {
    if (!id_out) return DDT_ERR_ARG;
    const NcclApi* n = nccl();
    if (!n) {
        set_error("libnccl.so.2 not found (import torch first, or set DDT_NCCL_LIB)");
        return DDT_ERR_UNSUPPORTED;
    }
    ncclUniqueIdMin id;
    int r = n->GetUniqueId(&id);
    if (r != 0) return nccl_fail("ncclGetUniqueId", r);
    std::memcpy(id_out, id.internal, sizeof(id.internal));
    return DDT_OK;
}

ddt_status_t ddt_nccl_comm_create(int32_t nranks, const void* id, int32_t rank, void** comm_out) {
    if (!id || !comm_out || nranks < 1 || rank < 0 || rank >= nranks) return DDT_ERR_ARG;
    const NcclApi* n = nccl();
    if (!n) {
        set_error("libnccl.so.2 not found");
        return DDT_ERR_UNSUPPORTED;
    }
    ncclUniqueIdMin uid;
    std::memcpy(uid.internal, id, sizeof(uid.internal));
    void* comm = nullptr;
    int r = n->CommInitRank(&comm, nranks, uid, rank);
    if (r != 0) return nccl_fail("ncclCommInitRank", r);
    *comm_out = comm;
    return DDT_OK;
}

ddt_status_t ddt_nccl_comm_destroy(void* comm) {
    if (!comm) return DDT_ERR_ARG;
    const NcclApi* n = nccl();
    if (!n) return DDT_ERR_UNSUPPORTED;
    int r = n->CommDestroy(comm);
    return r == 0 ? DDT_OK : nccl_fail("ncclCommDestroy", r);
}

ddt_status_t ddt_window_alloc(int device, int64_t bytes, void** ptr_out, void* ipc_handle_out) {
    if (!ptr_out || bytes <= 0) return DDT_ERR_ARG;
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(device);
    void* p = nullptr;
    cudaError_t e = cudaMalloc(&p, (size_t)bytes);
    if (e == cudaSuccess) e = cudaMemset(p, 0, (size_t)bytes);
    if (e == cudaSuccess && ipc_handle_out) {
        cudaIpcMemHandle_t h;
        e = cudaIpcGetMemHandle(&h, p);
        if (e == cudaSuccess) std::memcpy(ipc_handle_out, &h, sizeof(h));
    }
    if (prev >= 0) cudaSetDevice(prev);
    if (e != cudaSuccess) {
        if (p) cudaFree(p);
        return cuda_fail("window alloc", e);
    }
    *ptr_out = p;
    return DDT_OK;
}

ddt_status_t ddt_window_open(int device, const void* ipc_handle, void** ptr_out) {
    if (!ipc_handle || !ptr_out) return DDT_ERR_ARG;
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(device);
    cudaIpcMemHandle_t h;
    std::memcpy(&h, ipc_handle, sizeof(h));
    void* p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
    if (prev >= 0) cudaSetDevice(prev);
    if (e != cudaSuccess) return cuda_fail("cudaIpcOpenMemHandle", e);
    *ptr_out = p;
    return DDT_OK;
}

ddt_status_t ddt_window_close(void* peer_ptr) {
    if (!peer_ptr) return DDT_ERR_ARG;
    cudaError_t e = cudaIpcCloseMemHandle(peer_ptr);
    return e == cudaSuccess ? DDT_OK : cuda_fail("cudaIpcCloseMemHandle", e);
}

ddt_status_t ddt_window_free(void* ptr) {
    if (!ptr) return DDT_ERR_ARG;
    cudaError_t e = cudaFree(ptr);
    return e == cudaSuccess ? DDT_OK : cuda_fail("cudaFree(window)", e);
}

}  // extern "C"
