// pepp_internal.h — shared declarations inside libpepp_spmv.so (not installed).
#pragma once

#include "pepp_spmv.h"

#include <cstdint>
#include <vector>

#define PEPP_API __attribute__((visibility("default")))

// NVTX ranges around plan / exec / exchange / host calls (header-only NVTX3:
// a no-op unless a profiler injects itself, e.g. ncu --nvtx or nsys)
#include <nvtx3/nvToolsExt.h>
namespace pepp {
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};
}  // namespace pepp
#define PEPP_NVTX(name) ::pepp::NvtxRange pepp_nvtx_range_(name)

namespace pepp {

struct Welford {
    int64_t count = 0;
    double mean = 0.0;
    double m2 = 0.0;
    void add(double v);
};

pepp_history* history_new();
void history_free(pepp_history* h);
void history_add(pepp_history* h, uint64_t key, int32_t cand, double us);
const Welford* history_get(const pepp_history* h, uint64_t key, int32_t cand);
constexpr double kAbandonFactor = 4.0;   // calibration stops sampling a candidate this much slower than the best
double history_best_mean(const pepp_history* h, uint64_t key, int32_t ncand, const uint8_t* eligible);
bool history_abandoned(const Welford* w, double best_mean);
// refinement: after min_samples rounds, candidates whose mean is within
// kContendFactor of the best get rounds up to kRefineRounds x min_samples
constexpr double kContendFactor = 1.10;
constexpr int32_t kRefineRounds = 3;
bool history_contender(const Welford* w, double best_mean);
int32_t history_pick(const pepp_history* h, uint64_t key, int32_t ncand, const uint8_t* eligible,
                     int32_t min_samples, int32_t* calibrating, double* predicted_us);
// distribution choice (P and exchange): argmin of the agreed (max over ranks) means
int32_t dist_argmin(int32_t nd, const double* agreed, const uint8_t* eligible);
uint64_t context_key(int64_t nrows, int64_t ncols, int64_t nnz, double cv, int32_t nparts, int32_t instance);
bool history_prior(const pepp_history* h, uint64_t key, int32_t n, const int32_t* ids, double* prior,
                   uint64_t* from_key);
void halo_ghost_list(const int32_t* col, int64_t nnz, int64_t lo, int64_t hi, std::vector<int32_t>& out);

// last CUDA failure of this thread (pepp_last_error): message, failing expression, plan.cu line
void set_last_error(const char* msg, const char* expr, int line);

// ---- smart containers (containers.cu) ----
int64_t vector_length(const pepp_vector_t* v);
bool vector_simulated(const pepp_vector_t* v);

// ---- NCCL, loaded on demand with dlopen (nccl_dl.cpp) ----
// Only the handful of entry points the exchange needs; types mirror nccl.h
// (NCCL 2.x ABI). No link-time dependency, so the library loads (and its
// host-only utilities run) on machines without NCCL or a GPU.
typedef struct ncclComm_opaque* ncclComm_t;
typedef struct { char internal[128]; } ncclUniqueId;
enum { NCCL_INT8 = 0, NCCL_INT32 = 2, NCCL_INT64 = 4, NCCL_FLOAT32 = 7, NCCL_FLOAT64 = 8 };
enum { NCCL_OP_MAX = 2 };
struct Nccl {
    int (*GetUniqueId)(ncclUniqueId*);
    int (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int);
    int (*CommDestroy)(ncclComm_t);
    int (*CommGetAsyncError)(ncclComm_t, int*);
    const char* (*GetErrorString)(int);
    int (*GroupStart)();
    int (*GroupEnd)();
    int (*Send)(const void*, size_t, int, int, ncclComm_t, void*);
    int (*Recv)(void*, size_t, int, int, ncclComm_t, void*);
    int (*Broadcast)(const void*, void*, size_t, int, int, ncclComm_t, void*);
    int (*AllReduce)(const void*, void*, size_t, int, int, ncclComm_t, void*);
};
const Nccl* nccl_load();                   // nullptr if libnccl cannot be loaded

}  // namespace pepp
