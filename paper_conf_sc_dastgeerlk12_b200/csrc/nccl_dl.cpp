// nccl_dl.cpp — NCCL loaded on demand (dlopen), used only for partitioned
// calls (nranks > 1): the exchange step that makes one rank's y slice part
// of every other rank's next x (§IV-F's concatenation of
// sub-task outputs, P@27875, moved between B200s over NVLink / NVSwitch).
#include "pepp_internal.h"

#include <cuda_runtime.h>
#include <dlfcn.h>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

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

extern "C" PEPP_API pepp_status_t pepp_nccl_selftest(int32_t device) {
    const pepp::Nccl* n = pepp::nccl_load();
    if (!n) return PEPP_E_NCCL;
    int prev = -1;
    if (cudaGetDevice(&prev) != cudaSuccess) { (void)cudaGetLastError(); return PEPP_E_CUDA; }
    if (device >= 0 && cudaSetDevice(device) != cudaSuccess) { (void)cudaGetLastError(); return PEPP_E_CUDA; }
    pepp_status_t st = PEPP_OK;
    pepp::ncclComm_t comm = nullptr;
    cudaStream_t s = nullptr;
    constexpr int kN = 1000;
    const int dtypes[4] = {pepp::NCCL_INT32, pepp::NCCL_INT64, pepp::NCCL_FLOAT32, pepp::NCCL_FLOAT64};
    const size_t dsz[4] = {4, 8, 4, 8};
    void* d_src[4] = {nullptr, nullptr, nullptr, nullptr};
    void* d_dst[4] = {nullptr, nullptr, nullptr, nullptr};
    std::vector<unsigned char> h_src(kN * 8), h_dst(kN * 8);
    for (int i = 0; i < kN * 8; ++i) h_src[i] = (unsigned char)(i * 131 + 7);
    auto cuda_ok = [&](cudaError_t e) { if (e != cudaSuccess) { (void)cudaGetLastError(); if (!st) st = PEPP_E_CUDA; } return e == cudaSuccess; };
    auto nccl_ok = [&](int r) { if (r != 0 && !st) st = PEPP_E_NCCL; return r == 0; };
    pepp::ncclUniqueId id;
    if (cuda_ok(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking)) && nccl_ok(n->GetUniqueId(&id)) &&
        nccl_ok(n->CommInitRank(&comm, 1, id, 0))) {
        for (int t = 0; t < 4 && !st; ++t) {
            cuda_ok(cudaMalloc(&d_src[t], kN * dsz[t]));
            cuda_ok(cudaMalloc(&d_dst[t], kN * dsz[t]));
            if (!st) cuda_ok(cudaMemcpy(d_src[t], h_src.data(), kN * dsz[t], cudaMemcpyHostToDevice));
            if (!st) cuda_ok(cudaMemset(d_dst[t], 0, kN * dsz[t]));
        }
        // grouped send / recv to self, every value type the exchange uses
        if (!st && nccl_ok(n->GroupStart())) {
            for (int t = 0; t < 4; ++t) {
                nccl_ok(n->Send(d_src[t], kN, dtypes[t], 0, comm, s));
                nccl_ok(n->Recv(d_dst[t], kN, dtypes[t], 0, comm, s));
            }
            nccl_ok(n->GroupEnd());
        }
        // in-place broadcast (allgatherv slices) and max all-reduce (plan-time agreement)
        if (!st) nccl_ok(n->Broadcast(d_dst[3], d_dst[3], kN, pepp::NCCL_FLOAT64, 0, comm, s));
        if (!st) nccl_ok(n->AllReduce(d_dst[1], d_dst[1], kN, pepp::NCCL_INT64, pepp::NCCL_OP_MAX, comm, s));
        if (!st) cuda_ok(cudaStreamSynchronize(s));
        int async_err = 0;
        if (!st) { nccl_ok(n->CommGetAsyncError(comm, &async_err)); if (async_err) st = PEPP_E_NCCL; }
        for (int t = 0; t < 4 && !st; ++t) {
            if (!cuda_ok(cudaMemcpy(h_dst.data(), d_dst[t], kN * dsz[t], cudaMemcpyDeviceToHost))) break;
            if (std::memcmp(h_dst.data(), h_src.data(), kN * dsz[t]) != 0) st = PEPP_E_NCCL;
        }
    }
    if (comm) n->CommDestroy(comm);
    for (int t = 0; t < 4; ++t) { if (d_src[t]) cudaFree(d_src[t]); if (d_dst[t]) cudaFree(d_dst[t]); }
    if (s) cudaStreamDestroy(s);
    (void)cudaGetLastError();
    if (prev >= 0) cudaSetDevice(prev);
    return st;
}
