#include "nccl_loader.hpp"

#include <dlfcn.h>

#include <mutex>

#include "../common.hpp"

namespace fpm {

const NcclApi& nccl() {
    static NcclApi api;
    static bool ok = false;
    static std::once_flag once;
    static std::string why;
    std::call_once(once, [] {
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            why = dlerror() ? dlerror() : "dlopen failed";
            return;
        }
        auto sym = [&](const char* n) { return dlsym(h, n); };
#define FPM_NCCL_SYM(field, name)                                              \
    api.field = reinterpret_cast<decltype(api.field)>(sym(name));              \
    if (!api.field) {                                                          \
        why = std::string("missing symbol ") + name;                           \
        return;                                                                \
    }
        FPM_NCCL_SYM(GetUniqueId, "ncclGetUniqueId")
        FPM_NCCL_SYM(CommInitRank, "ncclCommInitRank")
        FPM_NCCL_SYM(CommInitRankConfig, "ncclCommInitRankConfig")
        FPM_NCCL_SYM(CommCount, "ncclCommCount")
        FPM_NCCL_SYM(CommAbort, "ncclCommAbort")
        FPM_NCCL_SYM(CommSplit, "ncclCommSplit")
        FPM_NCCL_SYM(CommDestroy, "ncclCommDestroy")
        FPM_NCCL_SYM(CommGetAsyncError, "ncclCommGetAsyncError")
        FPM_NCCL_SYM(GroupStart, "ncclGroupStart")
        FPM_NCCL_SYM(GroupEnd, "ncclGroupEnd")
        FPM_NCCL_SYM(Send, "ncclSend")
        FPM_NCCL_SYM(Recv, "ncclRecv")
        FPM_NCCL_SYM(Broadcast, "ncclBroadcast")
        FPM_NCCL_SYM(GetErrorString, "ncclGetErrorString")
#undef FPM_NCCL_SYM
        ok = true;
    });
    if (!ok) fail(FPM_ENCCL, "NCCL unavailable: %s", why.c_str());
    return api;
}

}  // namespace fpm
