// nccl_min.h -- the handful of NCCL entry points libddt uses, declared with
// the ABI of nccl.h 2.28 (torch-bundled copy) and resolved with dlsym.
#pragma once
#include <cstddef>

namespace ddt {

struct ncclUniqueIdMin {
    char internal[128];
};

// ncclDataType_t: ncclUint8 = 1 (nccl.h: ncclInt8=0, ncclChar=0, ncclUint8=1)
constexpr int kNcclUint8 = 1;
constexpr int kNcclInt32 = 2;   // ncclInt32
constexpr int kNcclInt64 = 4;   // ncclInt64
constexpr int kNcclMin = 3;     // ncclRedOp_t: ncclSum=0, ncclProd=1, ncclMax=2, ncclMin=3

struct NcclApi {
    bool ok = false;
    int (*GetUniqueId)(ncclUniqueIdMin*) = nullptr;
    int (*CommInitRank)(void** comm, int nranks, ncclUniqueIdMin id, int rank) = nullptr;
    int (*CommDestroy)(void* comm) = nullptr;
    int (*Send)(const void* buf, size_t count, int dtype, int peer, void* comm, void* stream) = nullptr;
    int (*Recv)(void* buf, size_t count, int dtype, int peer, void* comm, void* stream) = nullptr;
    int (*AllReduce)(const void* sb, void* rb, size_t count, int dtype, int op, void* comm, void* stream) = nullptr;
    int (*GroupStart)() = nullptr;
    int (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(int) = nullptr;
    int (*CommGetAsyncError)(void* comm, int* err) = nullptr;
};

const NcclApi* nccl();
}  // namespace ddt
