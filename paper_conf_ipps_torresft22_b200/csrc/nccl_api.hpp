// nccl_api.hpp -- the few NCCL entry points the SOMIER_EXCHANGE_NCCL route
// uses ("ncclGroupStart; ncclSend/ncclRecv x2; ncclGroupEnd"),
// resolved at run time with dlopen so that libsomier.so does not link NCCL:
// SOMIER_NCCL_LIB names the library (torch.distributed's own libnccl.so.2, set
// by the Python binding), else the system libnccl.so.2. Types are declared
// here with NCCL's ABI (nccl.h): a 128-byte unique id, opaque communicators,
// int results, ncclUint8 = 1.
#pragma once
#include <cuda_runtime.h>

#include <cstddef>
#include <string>

namespace paper {

struct NcclUniqueId {
    char internal[128];
};
using ncclComm = void*;

struct NcclLib {
    bool ok = false;
    std::string error;
    int (*GetUniqueId)(NcclUniqueId*) = nullptr;
    int (*CommInitRank)(ncclComm*, int, NcclUniqueId, int) = nullptr;
    int (*CommInitAll)(ncclComm*, int, const int*) = nullptr;
    int (*CommDestroy)(ncclComm) = nullptr;
    int (*Send)(const void*, size_t, int, int, ncclComm, cudaStream_t) = nullptr;
    int (*Recv)(void*, size_t, int, int, ncclComm, cudaStream_t) = nullptr;
    int (*GroupStart)() = nullptr;
    int (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(int) = nullptr;
};

constexpr int kNcclUint8 = 1;

// Loaded once per process; .ok false (and .error set) if unavailable.
const NcclLib& nccl_lib();

}  // namespace paper
