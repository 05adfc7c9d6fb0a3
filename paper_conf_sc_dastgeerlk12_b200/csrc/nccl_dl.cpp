// nccl_dl.cpp — NCCL loaded on demand (dlopen), used only for partitioned
// calls (nranks > 1): the exchange step that makes one rank's y slice part
// of every other rank's next x (§IV-F's concatenation of
// sub-task outputs, P@27875, moved between B200s over NVLink / NVSwitch).
#include "pepp_internal.h"

#include <dlfcn.h>
#include <cstdlib>
#include <mutex>

namespace pepp {

static Nccl g_nccl;
static bool g_loaded = false;
static std::once_flag g_once;

const Nccl* nccl_load() {
    std::call_once(g_once, [] {
        // PEPP_NCCL_LIB (an explicit path) wins — tests point it at a
        // same-ABI stand-in (tests/support/fake_nccl.c) to run several ranks
        // on one GPU; else the copy already mapped into the process (torch's),
        // then the system one.
        const char* names[] = {"libnccl.so.2", "libnccl.so"};
        void* h = nullptr;
        if (const char* path = std::getenv("PEPP_NCCL_LIB")) h = dlopen(path, RTLD_NOW | RTLD_LOCAL);
        for (int i = 0; !h && i < 2; ++i) h = dlopen(names[i], RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
        for (int i = 0; !h && i < 2; ++i) h = dlopen(names[i], RTLD_NOW | RTLD_GLOBAL);
        if (!h) return;
#define PEPP_SYM(field, name) g_nccl.field = reinterpret_cast<decltype(g_nccl.field)>(dlsym(h, name)); if (!g_nccl.field) return;
        PEPP_SYM(GetUniqueId, "ncclGetUniqueId")
        PEPP_SYM(CommInitRank, "ncclCommInitRank")
        PEPP_SYM(CommDestroy, "ncclCommDestroy")
        PEPP_SYM(CommGetAsyncError, "ncclCommGetAsyncError")
        PEPP_SYM(GetErrorString, "ncclGetErrorString")
        PEPP_SYM(GroupStart, "ncclGroupStart")
        PEPP_SYM(GroupEnd, "ncclGroupEnd")
        PEPP_SYM(Send, "ncclSend")
        PEPP_SYM(Recv, "ncclRecv")
        PEPP_SYM(Broadcast, "ncclBroadcast")
        PEPP_SYM(AllReduce, "ncclAllReduce")
#undef PEPP_SYM
        g_loaded = true;
    });
    return g_loaded ? &g_nccl : nullptr;
}

}  // namespace pepp

extern "C" PEPP_API pepp_status_t pepp_nccl_unique_id(void* id_out) {
    if (!id_out) return PEPP_E_INVALID;
    const pepp::Nccl* n = pepp::nccl_load();
    if (!n) return PEPP_E_NCCL;
    return n->GetUniqueId(reinterpret_cast<pepp::ncclUniqueId*>(id_out)) == 0 ? PEPP_OK : PEPP_E_NCCL;
}
