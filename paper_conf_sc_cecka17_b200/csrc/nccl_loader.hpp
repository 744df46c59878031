// nccl_loader.hpp — NCCL resolved at run time (dlopen "libnccl.so.2"), so the library loads
// without NCCL for G = 1 and shares the process's NCCL (e.g. torch's) when one is loaded.
#pragma once
#include <dlfcn.h>
#include <nccl.h>
#include <mutex>
#include <string>

namespace fmmfft {

struct NcclApi {
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
    bool ok = false;
    std::string err;
};

inline NcclApi& nccl() {
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        const char* names[] = {"libnccl.so.2", "libnccl.so"};
        void* h = nullptr;
        for (const char* n : names) {
            h = dlopen(n, RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);   // prefer an already-loaded NCCL
            if (!h) h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
            if (h) break;
        }
        if (!h) { api.err = std::string("dlopen libnccl.so.2 failed: ") + dlerror(); return; }
#define FMM_SYM(field, name)                                                         \
        api.field = reinterpret_cast<decltype(api.field)>(dlsym(h, name));           \
        if (!api.field) { api.err = std::string("missing NCCL symbol ") + name; return; }
        FMM_SYM(GetUniqueId, "ncclGetUniqueId")
        FMM_SYM(CommInitRank, "ncclCommInitRank")
        FMM_SYM(CommDestroy, "ncclCommDestroy")
        FMM_SYM(Send, "ncclSend")
        FMM_SYM(Recv, "ncclRecv")
        FMM_SYM(AllGather, "ncclAllGather")
        FMM_SYM(GroupStart, "ncclGroupStart")
        FMM_SYM(GroupEnd, "ncclGroupEnd")
        FMM_SYM(GetErrorString, "ncclGetErrorString")
#undef FMM_SYM
        api.ok = true;
    });
    return api;
}

}  // namespace fmmfft
