#include "nccl_dl.h"

#include <dlfcn.h>

#include <cstdlib>
#include <string>

namespace accmg {

NcclApi* nccl_api(const char** why) {
    static NcclApi api;
    static bool tried = false;
    static std::string err;
    if (tried) {
        if (!api.loaded && why) *why = err.c_str();
        return api.loaded ? &api : nullptr;
    }
    tried = true;
    void* h = nullptr;
    // 1. an NCCL already mapped into the process (torch's); 2. ACCMG_NCCL_PATH; 3. the loader path
    h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) {
        const char* p = std::getenv("ACCMG_NCCL_PATH");
        if (p) h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
    }
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
        err = std::string("cannot load libnccl.so.2: ") + dlerror();
        if (why) *why = err.c_str();
        return nullptr;
    }
#define LOAD(f)                                                        \
    api.f = reinterpret_cast<decltype(api.f)>(dlsym(h, "nccl" #f));    \
    if (!api.f) {                                                      \
        err = "NCCL symbol missing: nccl" #f;                          \
        if (why) *why = err.c_str();                                   \
        return nullptr;                                                \
    }
    LOAD(GetUniqueId) LOAD(CommInitRank) LOAD(CommDestroy) LOAD(GroupStart) LOAD(GroupEnd) LOAD(Send)
    LOAD(Recv) LOAD(AllReduce) LOAD(AllGather) LOAD(GetErrorString)
#undef LOAD
    api.loaded = true;
    return &api;
}

}  // namespace accmg
