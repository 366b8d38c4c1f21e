// nccl_api.h -- NCCL entry points loaded at run time (dlopen "libnccl.so.2").
//
// The library-owned communicator of afmm_p2p_config.nccl_id (rows a4/a8 of
// SURVEY.md S8(a)).  NCCL is not a link-time dependency: the .so loads (and
// every non-NCCL call works) on a box without NCCL, and in a process that
// already loaded libnccl.so.2 (torch.distributed) the same copy is reused
// (RTLD_NOLOAD first), so torch and the library never run two NCCL builds.
// Types and constants come from the NCCL header (ncclUniqueId, ncclComm_t,
// ncclConfig_t, the data type / reduction enums); only the functions are
// resolved by name.
#pragma once
#include <dlfcn.h>

#include <cstdlib>
#include <mutex>

#include <nccl.h>

namespace afmm {

struct NcclApi {
    bool ok = false;
    int version = 0;
    ncclResult_t (*GetVersion)(int *) = nullptr;
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommInitRankConfig)(ncclComm_t *, int, ncclUniqueId, int, ncclConfig_t *) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*CommAbort)(ncclComm_t) = nullptr;        // optional: destroy of a poisoned handle
    ncclResult_t (*Broadcast)(const void *, void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;
};

// The process-wide NCCL entry points (loaded once); api().ok == false when no
// libnccl.so.2 can be loaded.  AFMM_NCCL_LIB overrides the library path.
inline const NcclApi &nccl_api() {
    static NcclApi a;
    static std::once_flag once;
    std::call_once(once, [] {
        const char *path = getenv("AFMM_NCCL_LIB");
        void *lib = path ? dlopen(path, RTLD_NOW | RTLD_LOCAL) : dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
        if (!lib && !path) lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_LOCAL);
        if (!lib) return;
        auto sym = [&](const char *n) { return dlsym(lib, n); };
        a.GetVersion = reinterpret_cast<decltype(a.GetVersion)>(sym("ncclGetVersion"));
        a.GetUniqueId = reinterpret_cast<decltype(a.GetUniqueId)>(sym("ncclGetUniqueId"));
        a.CommInitRank = reinterpret_cast<decltype(a.CommInitRank)>(sym("ncclCommInitRank"));
        a.CommInitRankConfig = reinterpret_cast<decltype(a.CommInitRankConfig)>(sym("ncclCommInitRankConfig"));
        a.CommDestroy = reinterpret_cast<decltype(a.CommDestroy)>(sym("ncclCommDestroy"));
        a.CommAbort = reinterpret_cast<decltype(a.CommAbort)>(sym("ncclCommAbort"));
        a.Broadcast = reinterpret_cast<decltype(a.Broadcast)>(sym("ncclBroadcast"));
        a.AllReduce = reinterpret_cast<decltype(a.AllReduce)>(sym("ncclAllReduce"));
        a.GetErrorString = reinterpret_cast<decltype(a.GetErrorString)>(sym("ncclGetErrorString"));
        a.ok = a.GetVersion && a.GetUniqueId && a.CommInitRank && a.CommDestroy && a.Broadcast && a.AllReduce &&
               a.GetErrorString;
        if (a.ok) a.GetVersion(&a.version);
    });
    return a;
}

}  // namespace afmm
