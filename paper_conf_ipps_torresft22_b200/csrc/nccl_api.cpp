// nccl_api.cpp -- dlopen of NCCL for the SOMIER_EXCHANGE_NCCL route (see nccl_api.hpp).
#include "nccl_api.hpp"

#include <dlfcn.h>

#include <cstdlib>
#include <mutex>
#include <type_traits>

namespace paper {

const NcclLib& nccl_lib() {
    static NcclLib lib;
    static std::once_flag once;
    std::call_once(once, [] {
        const char* path = std::getenv("SOMIER_NCCL_LIB");
        void* h = dlopen(path && path[0] ? path : "libnccl.so.2", RTLD_NOW | RTLD_LOCAL);
        if (!h) {
            lib.error = std::string("dlopen(") + (path && path[0] ? path : "libnccl.so.2") + "): " + dlerror();
            return;
        }
        bool all = true;
        auto sym = [&](auto& fn, const char* name) {
            fn = reinterpret_cast<std::remove_reference_t<decltype(fn)>>(dlsym(h, name));
            if (!fn) {
                all = false;
                if (lib.error.empty()) lib.error = std::string("NCCL symbol missing: ") + name;
            }
        };
        sym(lib.GetUniqueId, "ncclGetUniqueId");
        sym(lib.CommInitRank, "ncclCommInitRank");
        sym(lib.CommInitAll, "ncclCommInitAll");
        sym(lib.CommDestroy, "ncclCommDestroy");
        sym(lib.Send, "ncclSend");
        sym(lib.Recv, "ncclRecv");
        sym(lib.GroupStart, "ncclGroupStart");
        sym(lib.GroupEnd, "ncclGroupEnd");
        sym(lib.GetErrorString, "ncclGetErrorString");
        lib.ok = all;
    });
    return lib;
}

}  // namespace paper
