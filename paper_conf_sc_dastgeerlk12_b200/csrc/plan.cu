// plan.cu — pepp_spmv_plan / _select / _exec / _destroy (see include/pepp_spmv.h).
//
// Steps of the hot path:
//   a1 context extraction     -> rowptr_check_narrow_kernel (+ host CV)     [plan]
//   a2 partition              -> caller / pepp_partition_rows; ghosts here  [plan]
//   a3 variant preparation    -> SELL conversion (+ stencil / 16-bit index compression),
//                                merge tile search, CSR-stream item table     [plan]
//   a4 selection              -> select_choice: calibration rounds / argmin  [each call, host]
//   a5 SpMV kernel            -> kernels.cuh                                 [each call, device]
//   a6 exchange               -> NCCL allgatherv (grouped broadcasts) / halo [each call, P > 1]
//   a7 history update         -> lazily harvested CUDA events -> Welford     [each call, host]
#include "pepp_internal.h"
#include "kernels.cuh"

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_select.cuh>
#include <thrust/iterator/counting_iterator.h>

#include <algorithm>
#include <map>
#include <mutex>
#include <thread>
#include <tuple>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

namespace {

using pepp::Nccl;
using pepp::ncclComm_t;

constexpr int kBlock = 256;
constexpr int kSellCapMin = 64;       // hybrid SELL: floor of the cap (prepare_sell_long)
#ifndef PEPP_EXP_CHUNK_COST   // experiments only: build-time override (PEPP_NVCC_EXTRA=-DPEPP_EXP_CHUNK_COST=n)
#define PEPP_EXP_CHUNK_COST 4
#endif
constexpr int64_t kChunkCost = PEPP_EXP_CHUNK_COST;   // SELL per-chunk overhead in slot-equivalents (warp ranges, hybrid cap)
constexpr int64_t kSellMidMax = 1024; // hybrid rows up to this length: one warp each (sell_mid_kernel)
#ifndef PEPP_SLIST_F64
#define PEPP_SLIST_F64 1
#endif
constexpr bool kSlistF64 = PEPP_SLIST_F64;   // stencil list for fp64 plans too (sell_stencil_list)
#ifndef PEPP_SLIST_CONCURRENT
#define PEPP_SLIST_CONCURRENT 1
#endif
constexpr bool kSlistConcurrent = PEPP_SLIST_CONCURRENT;   // genlist walk on a second stream
constexpr int kMergeBlock = 256;
constexpr int kMergeIPT = 7;
constexpr int kMergeTile = kMergeBlock * kMergeIPT;
// warp-granular merge-path: tiles of 32 x kMergeWarpIPT items, kMergeWarps warps per CTA
constexpr int kMergeWarpIPT = 7;
constexpr int kMergeWarps = 8;
constexpr int kMergeWarpTile = 32 * kMergeWarpIPT;
constexpr int kMergeWarpParam = 1000 + kMergeWarpIPT;   // candidate param of the warp-granular kernel
constexpr int kTimingRing = 64;
// TMA CSR-stream: items of <= kStreamNB nonzeros / <= kStreamRMAX rows, kStreamStages-deep ring
constexpr int kStreamBlock = 256;
constexpr int kStreamStages = 2;   // 2 x 26.7 KB per CTA -> 4 CTAs (32 warps) per SM
constexpr int kStreamNB = 2048;
constexpr int kStreamRMAX = 512;
constexpr int kStreamVecMinLen = 64;   // items whose longest row exceeds this reduce warp-per-row
constexpr int kReserveSms = 2;         // SMs the interior sub-plan's persistent grid leaves to the exchange
constexpr int kP2PMaxBuf = 4;          // symmetric buffers per plan (pepp_spmv_p2p_buffers)

struct Candidate {
    int32_t variant;
    int32_t param;
};

struct TimingRec {
    cudaEvent_t start = nullptr, stop = nullptr;
    int32_t cand = -1;
    bool pending = false;
};

struct PeerXfer {            // halo traffic with one peer
    int32_t peer;
    int64_t count;
    int64_t contig_start;    // >= 0: the entries are y[contig_start, contig_start+count)
    int* d_idx = nullptr;    // else: global indices into y (device)
    void* d_buf = nullptr;   // pack / unpack buffer (value type)
};

// SELL tiles (sell_tile_kernel) of one kind: pattern chunks, or stencil
// chunks whose values stream (sell_build_tiles)
struct TileLayout {
    int4* d_tiles = nullptr;      // {first chunk, chunks << 5 | set id, value block / 32, 0}
    int ntiles = 0, grid = 0, rows = 0, stage = 0, vstage = 0;
    int64_t chunks = 0;           // chunks the tiles hold
    int64_t lines = 0;            // multi-line tiles among them
    size_t smem = 0;              // dynamic shared memory per CTA
    pepp::k::PatTiles tt{};
};

// Column-panel layout (PEPP_V_PANEL) for one panel width 2^lg
struct PanelLayout {
    int lg = 0, npanels = 0;
    int64_t npairs = 0;
    int* d_prow = nullptr;        // [npairs] row of each (row, panel) pair, panel-major, row order within a panel
    int* d_pstart = nullptr;      // [npairs + 1] first entry of each pair in pcol / pval
    int* d_pcol = nullptr;        // [nnz] columns, panel-major
    void* d_pval = nullptr;       // [nnz] values (plan value type)
    std::vector<int> poff;        // [npanels + 1] pair range of each panel
};

// Distribution candidates (opts.dist_select, §8(a) a4: P and exchange are
// timed choices). P' < nranks: ranks 0..P'-1 each compute the union of
// nranks/P' consecutive row blocks (shipped to them at plan time).
struct DistPart {
    int32_t parts = 0;
    std::vector<int64_t> bounds;             // [parts + 1] global row boundaries under P'
    pepp_spmv_plan_t* plan = nullptr;        // this rank's block under P' (rank < P'), else none
    std::vector<PeerXfer> recv_x, send_x;    // after a P' call: own rows + own ghosts from their P' owners
    std::vector<PeerXfer> recv_g, send_g;    // after a P' = nranks call: what a P' call reads (its block +
                                             // its ghosts) beyond own rows + own ghosts, from their owners
};
struct DistCand {
    int32_t parts;                           // P'
    int32_t ex;                              // PEPP_X_HALO / PEPP_X_ALLGATHER
};

}  // namespace

struct pepp_spmv_plan_s {
    pepp_spmv_opts_t opts{};
    int device = 0;
    int sm_count = 148;
    pepp_status_t sticky = PEPP_OK;

    int64_t nrows = 0, ncols = 0, nnz = 0, first = 0, row_offset = 0, global_rows = 0;
    int pad = 0;
    std::vector<int64_t> row_bounds;
    std::string history_path;

    // device CSR
    int* d_rp = nullptr;
    int* d_col = nullptr;
    void* d_val = nullptr;      // value_type elements (fp64 or fp32)
    int vt = PEPP_VALUE_F64;     // value type of the plan
    size_t esz = 8;              // bytes per value
    int64_t dev_bytes = 0;

    // SELL-C-σ
    int sell_sigma = 0;
    int nchunks = 0;
    int64_t sell_slots = 0;
    int64_t* d_chunk_ptr = nullptr;
    int* d_chunk_len = nullptr;
    int* d_rowlen = nullptr;
    int* d_perm = nullptr;
    int* d_scol = nullptr;
    int16_t* d_scol16 = nullptr;
    int* d_soff = nullptr;           // stencil-chunk slot offsets
    int64_t sell_const_chunks = 0;   // chunks stored as a pattern-table id (value + index compression)
    int* d_patlist = nullptr;        // σ = 1: pattern chunks as (chunk << 5 | id), phase A of the kernel
    int* d_genlist = nullptr;        // σ = 1: the other chunks, phase B
    int npatc = 0, ngen = 0;
    // pattern tiles (sell_tile_kernel<…, VALS = false>): runs of pattern chunks cut into
    // tiles whose x ranges are bulk-copied; the pattern chunks no tile holds
    // stay in d_patrest for phase A of the genlist walk
    TileLayout ptl;                  // pattern tiles
    int* d_patrest = nullptr;
    int npatrest = 0;
    TileLayout stl;                  // stencil tiles (values streamed) over the stencil list
    int2* d_strest = nullptr;        // stencil-list entries no tile holds (sell_slist_kernel)
    int nstrest = 0;
    int2* d_stlist = nullptr;        // σ = 1, values streamed: stencil-list entries (sell_slist_kernel)
    int nstc = 0, grid_slist = 0;
    bool slist_long = false;                     // an offset set longer than 8: the 16-slot instance
    cudaStream_t gside = nullptr;                // the genlist walk's stream (concurrent with the list kernel)
    cudaEvent_t ev_gfork = nullptr, ev_gjoin = nullptr;
    pepp::k::SellStencils stab{};    // the distinct offset sets of the stencil list (kernel parameter)
    pepp::k::SellPatterns<double> pat64{};   // the pattern table, passed by value to the SELL kernel
    pepp::k::SellPatterns<float> pat32{};
    int64_t sell_stencil_chunks = 0;
    int sell_cpw = 1;            // chunks per σ window (chunk order is transposed when > 1)
    int* d_sell_ws = nullptr;    // σ > 1: per-warp ranges of the transposed chunk order, equal slots
    int64_t sell_col16_chunks = 0;
    void* d_sval = nullptr;
    // hybrid SELL: rows longer than sell_cap are summed by sell_long_kernel
    int sell_cap = INT32_MAX;
    int nsell_seg = 0, nsell_long = 0;
    int4* d_sell_seg = nullptr;      // {row, k begin, k end, long-row index} per segment
    int2* d_sell_lrow = nullptr;     // {first segment, segments} per long row
    unsigned int* d_sell_cnt = nullptr;
    int nsell_mid = 0;
    int* d_sell_mid = nullptr;       // rows of cap < length <= kSellLongSeg: sell_mid_kernel, warp per row
    int64_t sell_long_nnz = 0;       // entries of the rows the mid / long-row kernels sum
    int64_t sell_bytes = 0;          // DRAM bytes one SELL call streams with this layout (layout_bytes)
    void* d_sell_part = nullptr;     // segment partials (8-byte slots)

    // column panels (x beyond L2)
    std::vector<PanelLayout> panels;

    // merge path
    int ntiles = 0;
    int2* d_tile = nullptr;
    int* d_carry_row = nullptr;
    void* d_carry_val = nullptr;   // carries are stored in the plan's value type (8 B slots)
    int nlongruns = 0, nlongruns_w = 0;
    int4* d_longruns = nullptr;
    int4* d_longruns_w = nullptr;
    int ntiles_w = 0;
    int2* d_tile_w = nullptr;
    int* d_carry_row_w = nullptr;
    void* d_carry_val_w = nullptr;

    // TMA CSR-stream
    int nitems = 0, nlong = 0, grid_stream = 0;
    int4* d_items = nullptr;
    int4* d_longrows = nullptr;
    void* d_stream_carry = nullptr;

    // occupancy-derived grids
    int grid_csr[6] = {0};   // per log2(TPR)
    int grid_sell = 0;

    // selection
    pepp_plan_info_t info{};
    std::vector<Candidate> cands;
    std::vector<uint8_t> eligible;
    pepp_history* hist = nullptr;
    uint64_t key = 0;
    int64_t ncalls = 0;
    bool calibrated = false;   // calibration (rounds + refinement) finished: exploit without rescanning

    // timing ring
    TimingRec ring[kTimingRing];
    int ring_head = 0;   // oldest pending
    int ring_count = 0;
    std::vector<int32_t> pending;   // timed calls in flight per candidate
    std::vector<uint8_t> warmed;    // per candidate: its warm-up call (first timed call, not recorded) is done
    std::vector<int32_t> uids;      // stable candidate identity in the history: variant << 20 | param
    std::vector<int64_t> cand_bytes;// per candidate: bytes its kernels move per call (layout as stored + x + y)
    std::vector<double> prior;      // cold-start means from the nearest recorded context (-1 = none)
    std::vector<int32_t> order;     // calibration order (predicted best first)
    std::vector<double> predicted;  // opts.predict per candidate (-1 = none)
    uint64_t prior_key = 0;

    // multi-GPU
    const Nccl* nccl = nullptr;
    ncclComm_t comm = nullptr;
    bool own_comm = false;
    int32_t exchange = PEPP_X_NONE;
    std::vector<PeerXfer> recv_x, send_x;

    // halo / interior overlap (opts.overlap): head [0, h), interior, tail [R - t, R)
    pepp_spmv_plan_t* sub[3] = {nullptr, nullptr, nullptr};
    int64_t sub_r0[3] = {0, 0, 0};
    cudaStream_t side = nullptr;                 // exchange stream (highest priority)
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    // scratch ordering across streams (scratch_acquire / scratch_release)
    cudaEvent_t ev_scratch = nullptr;
    cudaStream_t scratch_stream = nullptr;
    bool scratch_used = false;
    int reserve_sms = 0;                         // SMs a persistent grid leaves free (interior sub-plan)
    std::vector<int64_t> send_local;             // plan time: local rows the peers receive

    // fused peer-memory halo (PEPP_X_P2P, pepp_spmv_p2p_buffers)
    struct SendRange { int32_t peer; int64_t lo, hi; };   // local rows [lo, hi) some peer receives
    std::vector<SendRange> send_rng;             // plan time (setup_halo)
    int p2p_nbuf = 0;
    void* p2p_buf[kP2PMaxBuf] = {};              // this rank's symmetric buffers (global length)
    unsigned long long* d_sig = nullptr;         // signal block: ready[P], arrive[P], epoch, done
    int* h_err = nullptr;                        // host-mapped error flag (a peer never arrived)
    int* d_err = nullptr;
    std::vector<void*> p2p_opened;               // IPC mappings of peers' buffers / signal blocks
    int p2p_npush = 0;
    int64_t p2p_push_lo[pepp::k::kP2PMaxPush] = {}, p2p_push_hi[pepp::k::kP2PMaxPush] = {};
    void* p2p_push_dst[kP2PMaxBuf][pepp::k::kP2PMaxPush] = {};
    int p2p_nsend = 0, p2p_nrecv = 0;
    unsigned long long* p2p_ready_in[pepp::k::kP2PMaxPeers] = {};    // per send peer
    unsigned long long* p2p_arrive_out[pepp::k::kP2PMaxPeers] = {};  // per send peer
    unsigned long long* p2p_ready_out[pepp::k::kP2PMaxPeers] = {};   // per receive peer
    unsigned long long* p2p_arrive_in[pepp::k::kP2PMaxPeers] = {};   // per receive peer
    int p2p_grid = 1;
    unsigned long long p2p_timeout_ns = 20ull * 1000 * 1000 * 1000;

    // distribution choice (opts.dist_select)
    std::vector<DistPart> dparts;                // P' < nranks
    std::vector<DistCand> dcands;                // (P', exchange) candidates, P' = nranks first
    std::vector<double> dist_agreed;             // agreed (max over ranks) mean µs per candidate
    int dist_next = -1, dist_repl = -1;          // chosen for PEPP_Y_NEXT_INPUT / PEPP_Y_REPLICATED calls
    bool p2p_use = true;                         // registered buffers: the fused push won (or no choice made)
    double p2p_agreed = 0.0;
    uint64_t dist_key = 0;
    int64_t global_nnz = 0;

    // plan-owned x / y for pepp_spmv_exec_host (allocated on first use)
    void* d_hx = nullptr;
    void* d_hy = nullptr;
    // pepp_spmv_exec_host_batch: two slots of (x, y) device buffers, copy
    // streams and their events (created on first use)
    void* d_hb[4] = {};
    cudaStream_t cs_in = nullptr, cs_out = nullptr;
    cudaEvent_t ev_start = nullptr, ev_end = nullptr, ev_in[2] = {}, ev_out[2] = {}, ev_free[2] = {};
};

namespace {

#define PEPP_CUDA_TRY(expr)                                   \
    do {                                                      \
        cudaError_t _e = (expr);                              \
        if (_e != cudaSuccess) {                              \
            pepp::set_last_error(cudaGetErrorString(_e), #expr, __LINE__); \
            (void)cudaGetLastError();                         \
            return PEPP_E_CUDA;                               \
        }                                                     \
    } while (0)

double now_ms() {
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

// Every entry point works on the plan's device and leaves the caller's
// current device as it found it.
struct DeviceScope {
    int prev = -1;
    bool ok = false;
    explicit DeviceScope(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) { (void)cudaGetLastError(); prev = -1; }
        ok = prev == dev || cudaSetDevice(dev) == cudaSuccess;
        if (!ok) (void)cudaGetLastError();
    }
    ~DeviceScope() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
        (void)cudaGetLastError();
    }
};

// device buffer of `bytes` bytes owned by the plan (value-typed arrays)
pepp_status_t dalloc_bytes(pepp_spmv_plan_t* p, void** ptr, int64_t bytes) {
    *ptr = nullptr;
    if (bytes <= 0) bytes = 8;
    cudaError_t e = cudaMalloc(ptr, (size_t)bytes);
    if (e != cudaSuccess) { pepp::set_last_error(cudaGetErrorString(e), "cudaMalloc", __LINE__); (void)cudaGetLastError(); *ptr = nullptr; return e == cudaErrorMemoryAllocation ? PEPP_E_NOMEM : PEPP_E_CUDA; }
    p->dev_bytes += bytes;
    return PEPP_OK;
}

// plan-time scratch device buffer, freed on every exit path
template <typename T>
struct DevTmp {
    T* p = nullptr;
    DevTmp() = default;
    DevTmp(const DevTmp&) = delete;
    DevTmp& operator=(const DevTmp&) = delete;
    DevTmp(DevTmp&& o) noexcept : p(o.p) { o.p = nullptr; }
    ~DevTmp() { if (p) cudaFree(p); }
    cudaError_t alloc(size_t n) { return cudaMalloc((void**)&p, sizeof(T) * (n ? n : 1)); }
    T* release() { T* r = p; p = nullptr; return r; }
};

// Host -> device upload of a large pageable operand (the matrix at plan
// time). A plain cudaMemcpy from pageable memory runs at ~10 GB/s on the
// GPU boxes (the driver stages it through one pinned buffer with one CPU
// thread); registering the caller's pages costs more than it saves (4 GB:
// 0.85 s + 0.18 s to unregister against 0.39 s; tools/r2/h2d_probe.py).
// Here kStageThreads host threads each copy their own chunks into their own
// pair of pinned buffers (process-wide, allocated once) and issue the DMA on
// their own stream; `st` then waits for every worker stream. Small, device
// and already-pinned operands go straight through cudaMemcpyAsync.
constexpr size_t kStageChunk = 16u << 20, kStageMin = 64u << 20;
constexpr int kStageThreads = 8;
struct StagePool {
    std::mutex mu;
    std::vector<void*> buf;   // kStageThreads x 2 pinned chunks (never freed: process lifetime)
};
StagePool& stage_pool() {
    static StagePool* sp = new StagePool;
    return *sp;
}

pepp_status_t upload(void* dst, const void* src, size_t bytes, cudaMemcpyKind kind, cudaStream_t st) {
    if (!bytes) return PEPP_OK;
    cudaPointerAttributes at{};
    const bool pageable = kind == cudaMemcpyHostToDevice && cudaPointerGetAttributes(&at, src) == cudaSuccess &&
                          at.type == cudaMemoryTypeUnregistered;
    (void)cudaGetLastError();
    if (!pageable || bytes < kStageMin) return cudaMemcpyAsync(dst, src, bytes, kind, st) == cudaSuccess ? PEPP_OK : PEPP_E_CUDA;
    StagePool& sp = stage_pool();
    std::lock_guard<std::mutex> lock(sp.mu);   // one staged upload at a time per process
    if (sp.buf.empty()) {
        for (int i = 0; i < 2 * kStageThreads; ++i) {
            void* b = nullptr;
            if (cudaHostAlloc(&b, kStageChunk, cudaHostAllocDefault) != cudaSuccess) {
                (void)cudaGetLastError();
                for (void* q : sp.buf) cudaFreeHost(q);
                sp.buf.clear();
                return cudaMemcpyAsync(dst, src, bytes, kind, st) == cudaSuccess ? PEPP_OK : PEPP_E_CUDA;
            }
            sp.buf.push_back(b);
        }
    }
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return PEPP_E_CUDA;
    // the worker streams start after the work already queued on st (the
    // destination's memset)
    cudaEvent_t ev_start = nullptr;
    if (cudaEventCreateWithFlags(&ev_start, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventRecord(ev_start, st) != cudaSuccess)
        return PEPP_E_CUDA;
    const size_t nchunks = (bytes + kStageChunk - 1) / kStageChunk;
    std::vector<int> fail(kStageThreads, 0);
    std::vector<cudaStream_t> ws(kStageThreads, nullptr);
    auto work = [&](int w) {
        if (cudaSetDevice(dev) != cudaSuccess || cudaStreamCreateWithFlags(&ws[w], cudaStreamNonBlocking) != cudaSuccess ||
            cudaStreamWaitEvent(ws[w], ev_start, 0) != cudaSuccess) { fail[w] = 1; return; }
        cudaEvent_t ev[2] = {nullptr, nullptr};
        for (auto& e : ev)
            if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) { fail[w] = 1; return; }
        int k = 0;
        for (size_t c = (size_t)w; c < nchunks && !fail[w]; c += kStageThreads, ++k) {
            const int b = k & 1;
            if (k >= 2 && cudaEventSynchronize(ev[b]) != cudaSuccess) { fail[w] = 1; break; }   // buffer b free again
            const size_t off = c * kStageChunk, n = std::min(kStageChunk, bytes - off);
            void* pin = sp.buf[2 * w + b];
            std::memcpy(pin, (const char*)src + off, n);
            if (cudaMemcpyAsync((char*)dst + off, pin, n, cudaMemcpyHostToDevice, ws[w]) != cudaSuccess ||
                cudaEventRecord(ev[b], ws[w]) != cudaSuccess) fail[w] = 1;
        }
        // the pinned buffers are reused by the next upload: wait for this one's DMAs
        if (cudaStreamSynchronize(ws[w]) != cudaSuccess) fail[w] = 1;
        for (auto& e : ev) if (e) cudaEventDestroy(e);
    };
    std::vector<std::thread> th;
    for (int w = 0; w < kStageThreads; ++w) th.emplace_back(work, w);
    for (auto& t : th) t.join();
    bool bad = false;
    for (int w = 0; w < kStageThreads; ++w) {
        bad |= fail[w] != 0;
        if (ws[w]) cudaStreamDestroy(ws[w]);
    }
    cudaEventDestroy(ev_start);
    if (bad) { (void)cudaGetLastError(); return PEPP_E_CUDA; }
    return PEPP_OK;
}

template <typename T>
pepp_status_t dalloc(pepp_spmv_plan_t* p, T** ptr, int64_t n) {
    *ptr = nullptr;
    if (n <= 0) n = 1;
    cudaError_t e = cudaMalloc((void**)ptr, sizeof(T) * (size_t)n);
    if (e != cudaSuccess) { pepp::set_last_error(cudaGetErrorString(e), "cudaMalloc", __LINE__); (void)cudaGetLastError(); *ptr = nullptr; return e == cudaErrorMemoryAllocation ? PEPP_E_NOMEM : PEPP_E_CUDA; }
    p->dev_bytes += (int64_t)sizeof(T) * n;
    return PEPP_OK;
}

void free_plan(pepp_spmv_plan_t* p) {
    if (!p) return;
    if (p->device >= 0) cudaSetDevice(p->device);
    void* bufs[] = {p->d_rp, p->d_col, p->d_val, p->d_chunk_ptr, p->d_chunk_len, p->d_rowlen, p->d_perm,
                    p->d_scol, p->d_scol16, p->d_soff, p->d_sval, p->d_tile, p->d_carry_row, p->d_carry_val, p->d_hx, p->d_hy,
                    p->d_items, p->d_longrows, p->d_stream_carry, p->d_tile_w, p->d_carry_row_w, p->d_carry_val_w, p->d_longruns, p->d_longruns_w, p->d_sell_ws, p->d_patlist, p->d_genlist, p->ptl.d_tiles, p->stl.d_tiles, p->d_patrest, p->d_strest,
                    p->d_sell_seg, p->d_sell_lrow, p->d_sell_cnt, p->d_sell_part, p->d_sell_mid, p->d_stlist};
    for (void* b : bufs) if (b) cudaFree(b);
    for (auto* v : {&p->recv_x, &p->send_x})
        for (auto& t : *v) { if (t.d_idx) cudaFree(t.d_idx); if (t.d_buf) cudaFree(t.d_buf); }
    for (auto& pl : p->panels)
        for (void* b : {(void*)pl.d_prow, (void*)pl.d_pstart, (void*)pl.d_pcol, pl.d_pval}) if (b) cudaFree(b);
    for (auto& dp : p->dparts) {
        for (auto* v : {&dp.recv_x, &dp.send_x, &dp.recv_g, &dp.send_g})
            for (auto& t : *v) { if (t.d_idx) cudaFree(t.d_idx); if (t.d_buf) cudaFree(t.d_buf); }
        free_plan(dp.plan);
    }
    for (auto& r : p->ring) { if (r.start) cudaEventDestroy(r.start); if (r.stop) cudaEventDestroy(r.stop); }
    for (void* m : p->p2p_opened) cudaIpcCloseMemHandle(m);
    for (void* b : p->p2p_buf) if (b) cudaFree(b);
    if (p->d_sig) cudaFree(p->d_sig);
    if (p->h_err) cudaFreeHost(p->h_err);
    if (p->comm && p->own_comm && p->nccl) p->nccl->CommDestroy(p->comm);
    if (p->hist) pepp::history_free(p->hist);
    for (auto* q : p->sub) free_plan(q);
    if (p->ev_fork) cudaEventDestroy(p->ev_fork);
    if (p->ev_join) cudaEventDestroy(p->ev_join);
    if (p->ev_scratch) cudaEventDestroy(p->ev_scratch);
    if (p->ev_gfork) cudaEventDestroy(p->ev_gfork);
    if (p->ev_gjoin) cudaEventDestroy(p->ev_gjoin);
    if (p->gside) cudaStreamDestroy(p->gside);
    if (p->side) cudaStreamDestroy(p->side);
    for (void* b : p->d_hb) if (b) cudaFree(b);
    for (cudaEvent_t e : {p->ev_start, p->ev_end, p->ev_in[0], p->ev_in[1], p->ev_out[0], p->ev_out[1], p->ev_free[0], p->ev_free[1]})
        if (e) cudaEventDestroy(e);
    if (p->cs_in) cudaStreamDestroy(p->cs_in);
    if (p->cs_out) cudaStreamDestroy(p->cs_out);
    delete p;
}

int grid_for(const void* fn, int block, int64_t work_items, int items_per_block, int sms) {
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, block, 0) != cudaSuccess || occ < 1) occ = 1;
    (void)cudaGetLastError();
    const int64_t need = (work_items + items_per_block - 1) / items_per_block;
    const int64_t cap = (int64_t)sms * occ * 4;   // 4 resident waves, grid-stride beyond
    return (int)std::max<int64_t>(1, std::min(need, cap));
}

// ---------------------------------------------------------------- SELL prep
// σ > 1: cut the transposed chunk order (the kernel's chunk_of) into one
// contiguous range per warp of the grid with equal cost (slots + a per-chunk
// overhead), so that the few long chunks of every window do not pile up on
// the warps a cyclic stride would hand them to.
pepp_status_t sell_warp_ranges(pepp_spmv_plan_t* p) {
    const int nc = p->nchunks, cpw = p->sell_cpw;
    const int W = p->grid_sell * (kBlock / 32);
    std::vector<int> len(nc > 0 ? nc : 1);
    if (nc > 0) PEPP_CUDA_TRY(cudaMemcpy(len.data(), p->d_chunk_len, sizeof(int) * nc, cudaMemcpyDeviceToHost));
    const int nwin = nc / cpw, nfull = nwin * cpw;
    auto chunk_of = [&](int i) { return i < nfull ? (i % nwin) * cpw + i / nwin : i; };
    const int64_t kChunkOverhead = kChunkCost;   // descriptor + per-lane loads + y store, in slot-equivalents
    int64_t total = 0;
    for (int i = 0; i < nc; ++i) total += (len[chunk_of(i)] & pepp::k::kSellLenMask) + kChunkOverhead;
    std::vector<int> ws(W + 1, nc);
    ws[0] = 0;
    int64_t acc = 0;
    int w = 1;
    for (int i = 0; i < nc && w < W; ++i) {
        acc += (len[chunk_of(i)] & pepp::k::kSellLenMask) + kChunkOverhead;
        while (w < W && acc * W >= total * w) ws[w++] = i + 1;
    }
    pepp_status_t s;
    if ((s = dalloc(p, &p->d_sell_ws, W + 1))) return s;
    PEPP_CUDA_TRY(cudaMemcpy(p->d_sell_ws, ws.data(), sizeof(int) * (W + 1), cudaMemcpyHostToDevice));
    return PEPP_OK;
}

// SELL tiles (sell_tile_kernel, σ = 1 plans): a list of stencil chunks
// (pattern chunks of value-compressed plans, or the stencil list's chunks
// whose values stream), sorted by set id, chunk order within a set, is cut
// into tiles of consecutive chunks of one set, <= rows rows each. Per set the
// distinct offsets are grouped into clusters (gap <= kTileGap elements: one
// bulk copy of a few extra elements is cheaper than another copy); cluster c
// copies x[r0 + clo_c, r0 + clo_c + round16(nr + cext_c)) — clo_c rounded
// down to 16 B (r0 is a multiple of 32 rows, so the rounding is the same for
// every tile). Chunks whose rounded ranges would leave [0, ncols) are
// trimmed off a run's start / end into the caller's rest list. Stage = the
// largest set's clusters at `rows` rows (+ rows x longest set values when
// they stream); rows = the largest multiple of 32 (<= range bytes of x per
// cluster) whose S stages fit the shared-memory budget.
#ifndef PEPP_PTILE
#define PEPP_PTILE 1   // value-compressed plans: pattern tiles
#endif
#ifndef PEPP_STILE
#define PEPP_STILE 3   // values streamed: stencil tiles (bit 0: fp32 plans, bit 1: fp64 plans); config 4: fp32 340 -> 281 us, fp64 605 -> 553 us (same box)
#endif
#ifndef PEPP_PTILE_S
#define PEPP_PTILE_S 2   // stages, pattern tiles (multi-line tiles: K + W lines of 16 KB per stage)
#endif
#ifndef PEPP_STILE_S
#define PEPP_STILE_S 3   // stages, stencil tiles (values streamed)
#endif
#ifndef PEPP_PTILE_RANGE_KB
#define PEPP_PTILE_RANGE_KB 16   // x bytes per cluster range: rows per tile = 16 KB / value size (fewer if the stages do not fit)
#endif
#ifndef PEPP_STILE_RANGE_KB
#define PEPP_STILE_RANGE_KB 8
#endif
#ifndef PEPP_PTILE_BLOCK
#define PEPP_PTILE_BLOCK 288   // one producer warp + 8 consumer warps
#endif
#ifndef PEPP_PTILE_SMEM_KB
#define PEPP_PTILE_SMEM_KB 200   // per CTA
#endif
constexpr bool kPatTiles = PEPP_PTILE;
constexpr int kStencilTiles = PEPP_STILE;
constexpr int kPtileS = PEPP_PTILE_S, kStileS = PEPP_STILE_S, kPtileBlock = PEPP_PTILE_BLOCK;
constexpr int kTileGap = 64;
constexpr size_t kPtileSmemBudget = (size_t)PEPP_PTILE_SMEM_KB * 1024;
#ifndef PEPP_MTILE_K
#define PEPP_MTILE_K 3   // lines per multi-line pattern tile (< 2: off); tools/r2/gpu_mtile.sh, config 4 fp64 / fp32 µs:
                         // off 199.3 / 105.3; K=4, 8 KB lines, S=4 183.6 / 119.7; K=6 S=3 197.5 / 115.9;
                         // K=8 S=2 181.0 / 116.3; K=2, 16 KB 214.9 / 116.8; K=3, 16 KB, S=2 181.6 / 102.6 (kept)
#endif
#ifndef PEPP_MTILE_LINE_KB
#define PEPP_MTILE_LINE_KB 16   // x bytes per line (rows per line = 16 KB / value size)
#endif
constexpr int kMarchK = PEPP_MTILE_K, kMarchLineBytes = PEPP_MTILE_LINE_KB * 1024;
#ifndef PEPP_TILE_MIN_ROWS_VALS
#define PEPP_TILE_MIN_ROWS_VALS 768    // mean rows per tile below which a plan keeps the register path (values streamed)
#endif
#ifndef PEPP_TILE_MIN_ROWS_PAT
#define PEPP_TILE_MIN_ROWS_PAT 1536    // ... (pattern tiles)
#endif
constexpr int kTileMinRowsVals = PEPP_TILE_MIN_ROWS_VALS, kTileMinRowsPat = PEPP_TILE_MIN_ROWS_PAT;

#ifndef PEPP_TILE_SIDE_BPS
#define PEPP_TILE_SIDE_BPS 8   // blocks per SM (cap) of the walks beside a tile kernel; measured 1 / 2 / 8: vc config 4 207.5 / 197.9 / 197.0 us, fp32 list 293 / 282 / 282 us
#endif
#ifndef PEPP_EXP_TILE_SIDE
#define PEPP_EXP_TILE_SIDE 0   // experiments only: 1 = the side walks after the tile kernel on its stream, 2 = skipped (wrong y)
#endif
int tile_side_grid(const pepp_spmv_plan_t* p, int grid) {
    return std::max(1, std::min(grid, PEPP_TILE_SIDE_BPS * std::max(1, p->sm_count - p->reserve_sms)));
}

// warps per tile CTA walking the grid-edge chunks (0: a second kernel on the
// side stream); config 4 µs, one box, walkers 0 / 2 / 4 — values streamed
// fp64 571.6 / 556.3 / 557.6, fp32 291.5 / 275.6 / 276.5; pattern tiles fp64
// 187.6 / 196.3 / 172.7, fp32 116.3 / 140.4 / 99.8 (with few walkers the walk
// outlasts the short pattern-tile kernel); pattern-tile walkers 4 / 6 / 8:
// fp64 172.4 / 173.9 / 176.7 µs, 4096² 57.3 / 52.4 / 52.6 µs
#ifndef PEPP_TILE_WALKERS_S
#define PEPP_TILE_WALKERS_S 4   // stencil tiles (values streamed)
#endif
#ifndef PEPP_TILE_WALKERS_P
#define PEPP_TILE_WALKERS_P 6   // pattern tiles
#endif
template <bool VALS> constexpr int tile_walkers() { return VALS ? PEPP_TILE_WALKERS_S : PEPP_TILE_WALKERS_P; }
#ifndef PEPP_STILE_BLOCK
#define PEPP_STILE_BLOCK 416   // producer + 12 consumer warps for stencil tiles (values streamed): config 4 fp64 549-552 vs 561-564 us with 8 (3 alternating repeats, tools/r2/gpu_sblock.sh), fp32 equal
#endif
template <bool VALS> constexpr int tile_block() { return (VALS ? PEPP_STILE_BLOCK : kPtileBlock) + 32 * tile_walkers<VALS>(); }

template <int S, bool VALS, typename T>
const void* tile_kernel_fn() { return (const void*)pepp::k::sell_tile_kernel<tile_block<VALS>(), S, VALS, T, tile_walkers<VALS>()>; }

// ents[i] = {chunk, set id, value block / 32, -}; sorted by set id then chunk.
// Fills *L and appends the indices of untiled entries to *rest.
template <typename T>
pepp_status_t sell_build_tiles(pepp_spmv_plan_t* p, int nsets, const int* lens, const int (*offs)[pepp::k::kTileMaxLen],
                               const std::vector<int4>& ents, bool vals, TileLayout* L, std::vector<size_t>* rest) {
    using pepp::k::kTileMaxLen;
    constexpr int A = 16 / (int)sizeof(T);
    const int S = vals ? kStileS : kPtileS;
    const int range_bytes = (vals ? PEPP_STILE_RANGE_KB : PEPP_PTILE_RANGE_KB) * 1024;
    auto rdn = [](int64_t v) { return (v >= 0 ? v / A : -((-v + A - 1) / A)) * A; };
    auto rup = [](int64_t v) { return ((v + A - 1) / A) * A; };
    *L = TileLayout{};
    pepp::k::PatTiles tt{};
    if (nsets > pepp::k::kTileMaxSets) return PEPP_OK;
    int64_t emax = 0;
    int maxcl = 1, maxlen = 1;
    std::vector<std::pair<std::vector<int64_t>, std::vector<int64_t>>> clusters(nsets);
    for (int q = 0; q < nsets; ++q) {
        const int len = lens[q];
        if (len < 1 || len > kTileMaxLen) return PEPP_OK;
        tt.len[q] = len;
        maxlen = std::max(maxlen, len);
        std::vector<int> o(offs[q], offs[q] + len);
        std::sort(o.begin(), o.end());
        o.erase(std::unique(o.begin(), o.end()), o.end());
        std::vector<int64_t> lo, hi;
        for (int v : o) {
            if (!lo.empty() && (int64_t)v - hi.back() <= kTileGap) { hi.back() = v; continue; }
            lo.push_back(v);
            hi.push_back(v);
        }
        const int nc = (int)lo.size();
        tt.ncl[q] = nc;
        maxcl = std::max(maxcl, nc);
        clusters[q] = {lo, hi};
        int64_t extra = 0;
        for (int c = 0; c < nc; ++c) {
            const int64_t clo = rdn(lo[c]), cext = hi[c] - clo;
            if (clo < INT32_MIN / 2 || clo > INT32_MAX / 2 || cext > (1 << 20)) return PEPP_OK;   // no tiles
            tt.clo[q][c] = (int)clo;
            tt.cext[q][c] = (int)cext;
            extra += rup(cext) + A;   // round16(nr + cext) <= nr + round16(cext) (nr a multiple of 32)
        }
        emax = std::max(emax, extra);
    }
    // multi-line tiles (pattern tiles of grid stencils): per set, D = the
    // largest |cluster centre|, a_c = round(centre_c / D), b_c = lo_c - a_c·D;
    // usable when D keeps 16-B alignment, every |b_c| <= D / 4 and the lines
    // stay short (lext <= 4096) — e.g. 5- / 9-point 2-D (W = 2), 7-point 3-D
    // (D = n², ±n inside the line)
    std::vector<int> amin_of(nsets, 0);
    std::vector<std::vector<int>> a_of(nsets);
    bool march = !vals && kMarchK >= 2;
    int wmax = 0, lextmax = 0;
    for (int q = 0; q < nsets && march; ++q) {
        const auto& lo = clusters[q].first;
        const auto& hi = clusters[q].second;
        int64_t D = 0;
        for (size_t c = 0; c < lo.size(); ++c) D = std::max<int64_t>(D, std::llabs((lo[c] + hi[c]) / 2));
        tt.D[q] = 0;
        if (D < 64 || D % A || D > INT32_MAX / 8) continue;   // no line structure: regular tiles
        int amin = INT32_MAX, amax = INT32_MIN;
        int64_t bmin = INT64_MAX, bmax = INT64_MIN;
        bool ok = true;
        std::vector<int> a(lo.size());
        for (size_t c = 0; c < lo.size(); ++c) {
            const double ctr = 0.5 * (double)(lo[c] + hi[c]);
            a[c] = (int)std::llround(ctr / (double)D);
            const int64_t b = lo[c] - (int64_t)a[c] * D;
            ok &= std::llabs(b) <= D / 4;
            amin = std::min(amin, a[c]);
            amax = std::max(amax, a[c]);
            bmin = std::min(bmin, b);
            bmax = std::max(bmax, b + (hi[c] - lo[c]));
        }
        bmin = rdn(bmin);
        if (!ok || amax - amin > 4 || bmax - bmin > 4096) continue;
        tt.D[q] = (int)D;
        tt.W[q] = amax - amin;
        tt.lbase[q] = (int)((int64_t)amin * D + bmin);
        tt.lext[q] = (int)(bmax - bmin);
        amin_of[q] = amin;
        a_of[q] = a;
        wmax = std::max(wmax, tt.W[q]);
        lextmax = std::max(lextmax, tt.lext[q]);
    }
    if (march) {
        march = false;
        for (int q = 0; q < nsets; ++q) march |= tt.D[q] > 0;
    }
    // S stages (x ranges, + values) and barriers / entries within the budget;
    // with lines, rows per line = kMarchLineBytes of x and K + W lines per stage
    int rows = std::max(32, (march ? kMarchLineBytes : range_bytes) / (int)sizeof(T) / 32 * 32);
    auto xpart = [&](int r) { return rup((int64_t)maxcl * r + emax); };
    auto mpart = [&](int r) { return march ? (int64_t)(kMarchK + wmax) * rup(r + lextmax) : 0; };
    auto stage_of = [&](int r) { return std::max(xpart(r), mpart(r)) + (vals ? (int64_t)r * maxlen : 0); };
    while (rows >= 32 && (size_t)S * (size_t)stage_of(rows) * sizeof(T) + 32 * S + 64 > kPtileSmemBudget) rows -= 32;
    if (rows < 32 && march) {   // lines too long for K + W per stage (wide 3-D grids): single-line tiles
        march = false;
        for (int q = 0; q < nsets; ++q) tt.D[q] = 0;
        rows = std::max(32, range_bytes / (int)sizeof(T) / 32 * 32);
        while (rows >= 32 && (size_t)S * (size_t)stage_of(rows) * sizeof(T) + 32 * S + 64 > kPtileSmemBudget) rows -= 32;
    }
    if (rows < 32) return PEPP_OK;
    for (int q = 0; q < nsets && march; ++q) {
        if (!tt.D[q]) continue;
        tt.lws[q] = (int)rup(rows + lextmax);
        const auto& lo = clusters[q].first;
        for (int j = 0; j < tt.len[q]; ++j) {
            size_t c = 0;
            while (c + 1 < lo.size() && offs[q][j] >= lo[c + 1]) ++c;
            const int64_t a = a_of[q][c];
            tt.msidx[q][j] = (int)((a - amin_of[q]) * tt.lws[q] + (offs[q][j] - a * tt.D[q] - (tt.lbase[q] - (int64_t)amin_of[q] * tt.D[q])));
        }
    }
    for (int q = 0; q < nsets; ++q) {
        int64_t d = 0;
        for (int c = 0; c < tt.ncl[q]; ++c) { tt.cdst[q][c] = (int)d; d += rup(rows + tt.cext[q][c]); }
        for (int j = 0; j < tt.len[q]; ++j) {
            int c = 0;
            while (c + 1 < tt.ncl[q] && offs[q][j] >= tt.clo[q][c + 1]) ++c;
            tt.sidx[q][j] = tt.cdst[q][c] + (offs[q][j] - tt.clo[q][c]);
        }
    }
    // the tiles: runs of consecutive chunks of one set (their values are
    // consecutive too: σ = 1, chunk_ptr advances by 32 x len)
    std::vector<int4> tiles;
    const int cmax = rows / 32;
    // 0: fits; 1: a range starts below x[0]; 2: a range (or the rows) ends past the end
    auto misfit = [&](int64_t r0, int nr, int q) {
        if (r0 + nr > p->nrows) return 2;
        for (int c = 0; c < tt.ncl[q]; ++c) {
            const int64_t a = r0 + tt.clo[q][c], b = a + rup(nr + tt.cext[q][c]);
            if (a < 0) return 1;
            if (b > p->ncols) return 2;
        }
        return 0;
    };
    auto next_of = [&](size_t i, size_t k) {   // entry k continues entry i's run
        return ents[k].y == ents[i].y && (int64_t)ents[k].x == (int64_t)ents[i].x + (int64_t)(k - i) &&
               (!vals || (int64_t)ents[k].z == (int64_t)ents[i].z + (int64_t)(k - i) * tt.len[ents[i].y]);
    };
    int64_t tiled = 0;
    for (size_t i = 0; i < ents.size();) {
        const int q = ents[i].y;
        size_t j = i + 1;
        while (j < ents.size() && (int)(j - i) < cmax && next_of(i, j)) ++j;
        size_t a = i, b = j;
        for (int m; a < b && (m = misfit((int64_t)ents[a].x * 32, (int)(b - a) * 32, q)) != 0;) {
            if (m == 1) rest->push_back(a++);
            else rest->push_back(--b);
        }
        if (a < b) {
            tiles.push_back(make_int4(ents[a].x, ((int)(b - a) << 5) | q, ents[a].z, 0));
            tiled += (int64_t)(b - a);
        }
        i = j;
    }
    if (tiles.empty()) { rest->clear(); return PEPP_OK; }
    // tiles pay only on long runs (tools/r2/tile_vs_reg.py, tile / register
    // µs): 2-D Laplacians n = 512 / 1024 / 2048 / 4096 — values streamed 1.01 /
    // 0.74 / 0.88 / 0.87, value-compressed 1.35 / 1.21 / 0.82 / 0.69; 3-D
    // 7-point (5 clusters, runs of 2-8 chunks) 1.3-2.3. Short runs leave the
    // chunks to the register paths.
    if (tiled * 32 < (int64_t)tiles.size() * (vals ? kTileMinRowsVals : kTileMinRowsPat)) {
        rest->clear();
        return PEPP_OK;
    }
    if (march) {
        // columns: tiles of one set and length whose first rows differ by D,
        // cut into blocks of <= K lines; a block of >= 2 lines becomes one
        // multi-line tile when all its K + W lines lie inside x
        std::map<std::tuple<int, int, int64_t>, std::vector<size_t>> cols;
        for (size_t t = 0; t < tiles.size(); ++t) {
            const int q = tiles[t].y & 31;
            if (!tt.D[q]) continue;
            const int64_t r0 = (int64_t)tiles[t].x * 32;
            cols[{q, tiles[t].y >> 5, r0 % tt.D[q]}].push_back(t);
        }
        std::vector<uint8_t> absorbed(tiles.size(), 0);
        std::vector<int4> multi;
        for (auto& kv : cols) {
            auto& v = kv.second;   // ascending r0 (tiles are in chunk order within a set)
            const int q = std::get<0>(kv.first), nr = std::get<1>(kv.first) * 32;
            const int64_t D = tt.D[q];
            const int64_t lb = rup(nr + tt.lext[q]);
            for (size_t i = 0; i < v.size();) {
                size_t j = i + 1;
                while (j < v.size() && (int)(j - i) < kMarchK &&
                       (int64_t)tiles[v[j]].x * 32 == (int64_t)tiles[v[i]].x * 32 + (int64_t)(j - i) * D) ++j;
                const int K = (int)(j - i);
                const int64_t r0 = (int64_t)tiles[v[i]].x * 32;
                const int64_t a = r0 + tt.lbase[q], b = a + (int64_t)(K + tt.W[q] - 1) * D + lb;
                if (K >= 2 && a >= 0 && b <= p->ncols) {
                    multi.push_back(make_int4(tiles[v[i]].x, tiles[v[i]].y, K, 0));
                    for (size_t k = i; k < j; ++k) absorbed[v[k]] = 1;
                }
                i = j;
            }
        }
        if (!multi.empty()) {
            std::vector<int4> all;
            for (size_t t = 0; t < tiles.size(); ++t) if (!absorbed[t]) all.push_back(tiles[t]);
            all.insert(all.end(), multi.begin(), multi.end());
            // set, then first row: the grid's front advances through x together
            std::stable_sort(all.begin(), all.end(), [](const int4& u, const int4& w) {
                return (u.y & 31) != (w.y & 31) ? (u.y & 31) < (w.y & 31) : u.x < w.x;
            });
            tiles.swap(all);
            L->lines = (int64_t)multi.size();
        }
    }
    const size_t smem = (size_t)S * (size_t)stage_of(rows) * sizeof(T) + 32 * S;
    const void* fn = vals ? tile_kernel_fn<kStileS, true, T>() : tile_kernel_fn<kPtileS, false, T>();
    // the attribute is per kernel, not per plan: set the budget every plan's
    // tiles fit in (a plan setting its own, smaller size would make another
    // plan's launches of the same kernel fail)
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kPtileSmemBudget) != cudaSuccess) {
        (void)cudaGetLastError();   // the device cannot give a CTA that much shared memory: no tiles
        *L = TileLayout{};
        rest->clear();
        return PEPP_OK;
    }
    pepp_status_t s;
    if ((s = dalloc(p, &L->d_tiles, (int64_t)tiles.size()))) return s;
    PEPP_CUDA_TRY(cudaMemcpy(L->d_tiles, tiles.data(), sizeof(int4) * tiles.size(), cudaMemcpyHostToDevice));
    L->ntiles = (int)tiles.size();
    L->chunks = tiled;
    L->rows = rows;
    L->stage = (int)stage_of(rows);
    L->vstage = vals ? (int)xpart(rows) : 0;
    L->tt = tt;
    L->smem = smem;
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, vals ? tile_block<true>() : tile_block<false>(), L->smem) != cudaSuccess || occ < 1) occ = 1;
    (void)cudaGetLastError();
    L->grid = (int)std::max<int64_t>(1, std::min<int64_t>(L->ntiles, (int64_t)std::max(1, p->sm_count - p->reserve_sms) * occ));
    return PEPP_OK;
}

pepp_status_t ensure_side_stream(pepp_spmv_plan_t* p) {
    if (!kSlistConcurrent || p->gside) return PEPP_OK;
    PEPP_CUDA_TRY(cudaStreamCreateWithFlags(&p->gside, cudaStreamNonBlocking));
    PEPP_CUDA_TRY(cudaEventCreateWithFlags(&p->ev_gfork, cudaEventDisableTiming));
    PEPP_CUDA_TRY(cudaEventCreateWithFlags(&p->ev_gjoin, cudaEventDisableTiming));
    return PEPP_OK;
}

// pattern tiles from the pattern list (entries chunk << 5 | id); untiled
// entries -> d_patrest (phase A of the genlist walk)
template <typename T>
pepp_status_t sell_pattern_tiles(pepp_spmv_plan_t* p, const pepp::k::SellPatterns<T>& pt, const std::vector<int>& pat) {
    int npat = 0;
    for (int e : pat) npat = std::max(npat, (e & 31) + 1);
    int lens[pepp::k::kTileMaxSets] = {0};
    int offs[pepp::k::kTileMaxSets][pepp::k::kTileMaxLen] = {{0}};
    for (int q = 0; q < npat; ++q) {
        lens[q] = pt.len[q];
        for (int j = 0; j < pt.len[q]; ++j) offs[q][j] = pt.off[q][j];
    }
    std::vector<int4> ents(pat.size());
    for (size_t i = 0; i < pat.size(); ++i) ents[i] = make_int4(pat[i] >> 5, pat[i] & 31, 0, 0);
    std::vector<size_t> rest;
    pepp_status_t s;
    if ((s = sell_build_tiles<T>(p, npat, lens, offs, ents, false, &p->ptl, &rest))) return s;
    if (!p->ptl.ntiles) return PEPP_OK;
    std::sort(rest.begin(), rest.end());   // the pattern list's order (grouped by id)
    if (!rest.empty()) {
        std::vector<int> r(rest.size());
        for (size_t i = 0; i < rest.size(); ++i) r[i] = pat[rest[i]];
        if ((s = dalloc(p, &p->d_patrest, (int64_t)r.size()))) return s;
        PEPP_CUDA_TRY(cudaMemcpy(p->d_patrest, r.data(), sizeof(int) * r.size(), cudaMemcpyHostToDevice));
    }
    p->npatrest = (int)rest.size();
    if (p->ngen + p->npatrest > 0) return ensure_side_stream(p);
    return PEPP_OK;
}

// Value + index compression: constant stencil chunks (cflag) with the same
// (length, offsets, value bits) become one entry of the pattern table; the
// chunk keeps its length, trades kSellStencil for kSellPattern, and its
// chunk_ptr entry becomes the pattern id. At most kSellMaxPatterns patterns
// of at most kSellMaxPatternLen slots; other chunks stay as they are.
template <typename T>
pepp_status_t sell_patterns(pepp_spmv_plan_t* p, int64_t nsb, const void* d_sconst, const unsigned char* d_cflag,
                            pepp::k::SellPatterns<T>* pt) {
    using pepp::k::kSellLenMask;
    const int nc = p->nchunks;
    std::vector<unsigned char> cflag(nc);
    std::vector<int> clen(nc), soff(nsb);
    std::vector<int64_t> cp(nc + 1);
    std::vector<T> sval(nsb);
    PEPP_CUDA_TRY(cudaMemcpy(cflag.data(), d_cflag, nc, cudaMemcpyDeviceToHost));
    PEPP_CUDA_TRY(cudaMemcpy(clen.data(), p->d_chunk_len, sizeof(int) * nc, cudaMemcpyDeviceToHost));
    PEPP_CUDA_TRY(cudaMemcpy(cp.data(), p->d_chunk_ptr, sizeof(int64_t) * (nc + 1), cudaMemcpyDeviceToHost));
    PEPP_CUDA_TRY(cudaMemcpy(soff.data(), p->d_soff, sizeof(int) * nsb, cudaMemcpyDeviceToHost));
    PEPP_CUDA_TRY(cudaMemcpy(sval.data(), d_sconst, sizeof(T) * nsb, cudaMemcpyDeviceToHost));
    *pt = pepp::k::SellPatterns<T>{};
    int npat = 0;
    int64_t used = 0;
    for (int c = 0; c < nc; ++c) {
        if (!cflag[c]) continue;
        const int len = clen[c] & kSellLenMask;
        if (len < 1 || len > pepp::k::kSellMaxPatternLen) continue;
        const int64_t sb = cp[c] >> 5;
        int pid = -1;
        for (int q = 0; q < npat && pid < 0; ++q) {
            bool same = pt->len[q] == len;
            for (int j = 0; same && j < len; ++j)
                same = pt->off[q][j] == soff[sb + j] && std::memcmp(&pt->val[q][j], &sval[sb + j], sizeof(T)) == 0;
            if (same) pid = q;
        }
        if (pid < 0) {
            if (npat == pepp::k::kSellMaxPatterns) continue;
            pid = npat++;
            pt->len[pid] = len;
            for (int j = 0; j < len; ++j) { pt->off[pid][j] = soff[sb + j]; pt->val[pid][j] = sval[sb + j]; }
        }
        clen[c] = (clen[c] & ~pepp::k::kSellStencil) | pepp::k::kSellPattern;
        cp[c] = pid;
        ++used;
    }
    // value compression only where it covers most chunks: a minority of
    // pattern chunks would keep the plan off the stencil list / stencil tiles
    // for all its other stencil chunks (the list and the pattern table are
    // alternatives), which costs more than the few values it saves
    if (!used || 2 * used < (int64_t)nc) { *pt = pepp::k::SellPatterns<T>{}; return PEPP_OK; }
    PEPP_CUDA_TRY(cudaMemcpy(p->d_chunk_len, clen.data(), sizeof(int) * nc, cudaMemcpyHostToDevice));
    PEPP_CUDA_TRY(cudaMemcpy(p->d_chunk_ptr, cp.data(), sizeof(int64_t) * nc, cudaMemcpyHostToDevice));
    p->sell_const_chunks = used;
    if (!p->d_perm) {   // σ = 1: split the chunks into the kernel's two phases
        std::vector<int> pat, gen;
        pat.reserve(used);
        gen.reserve(nc - used);
        for (int c = 0; c < nc; ++c) {
            if (clen[c] & pepp::k::kSellPattern) pat.push_back((c << 5) | (int)cp[c]);
            else gen.push_back(c);
        }
        // grouped by pattern (the kernel reloads its register copy of the
        // pattern only when the id changes), chunk order within a pattern
        std::stable_sort(pat.begin(), pat.end(), [](int a, int b) { return (a & 31) < (b & 31); });
        pepp_status_t s;
        if ((s = dalloc(p, &p->d_patlist, (int64_t)pat.size()))) return s;
        if ((s = dalloc(p, &p->d_genlist, (int64_t)gen.size()))) return s;
        PEPP_CUDA_TRY(cudaMemcpy(p->d_patlist, pat.data(), sizeof(int) * pat.size(), cudaMemcpyHostToDevice));
        if (!gen.empty()) PEPP_CUDA_TRY(cudaMemcpy(p->d_genlist, gen.data(), sizeof(int) * gen.size(), cudaMemcpyHostToDevice));
        p->npatc = (int)pat.size();
        p->ngen = (int)gen.size();
        if (kPatTiles && (s = sell_pattern_tiles<T>(p, *pt, pat))) return s;
    }
    return PEPP_OK;
}

// Phase A of the value-compressed walk reads list entries k, k + W, k + 2W,
// k + 3W as one group (W = warps of the grid). Reordering the list so that
// those positions hold kPatU *consecutive* entries of the pattern-sorted
// list gives each group a contiguous run of 4 chunks (128 rows): the group's
// x reads per offset become one 1 KB run instead of four scattered 256 B
// ones. Any order is correct (each entry is processed once); entries past
// the last whole super-group keep their place.
#ifndef PEPP_PAT_INTERLEAVE
#define PEPP_PAT_INTERLEAVE 0   // measured neutral on config 4 (261.0 vs 261.3 us, two alternating repeats): off
#endif
constexpr bool kPatInterleave = PEPP_PAT_INTERLEAVE;

pepp_status_t sell_patlist_interleave(pepp_spmv_plan_t* p) {
    const int64_t n = p->npatc, W = (int64_t)p->grid_sell * (kBlock / 32), U = pepp::k::kPatU;
    const int64_t G = n / (U * W);   // whole super-groups
    if (G == 0) return PEPP_OK;
    std::vector<int> src(n), dst(n);
    PEPP_CUDA_TRY(cudaMemcpy(src.data(), p->d_patlist, sizeof(int) * n, cudaMemcpyDeviceToHost));
    for (int64_t g = 0; g < G; ++g)
        for (int64_t w = 0; w < W; ++w)
            for (int64_t u = 0; u < U; ++u) dst[g * U * W + u * W + w] = src[(g * W + w) * U + u];
    for (int64_t i = G * U * W; i < n; ++i) dst[i] = src[i];
    PEPP_CUDA_TRY(cudaMemcpy(p->d_patlist, dst.data(), sizeof(int) * n, cudaMemcpyHostToDevice));
    return PEPP_OK;
}

// Hybrid SELL for heavy-tailed rows. One warp walks a whole chunk, so a
// chunk of L slots is a chain of L dependent slot steps on one warp, and in a
// sorted window the chunk holding the window's longest rows is padded to its
// longest row with mostly masked lanes. Rows longer than
//   cap = max(kSellCapMin, min(share, 8 x mean)),
// share = one warp's part of the SELL work ((nnz/32 + kChunkCost x chunks) /
// warps of one resident wave), leave the layout: up to kSellMidMax entries
// one warp each (sell_mid_kernel), longer ones cut into segments of
// kSellLongSeg for sell_long_kernel. Measured (tools/gpu_cap4.sh, `skew` /
// config 3, µs): cap 1024 and no mid kernel 373 / 359; share 276 / 359;
// 128 241 / 352; 64 236 / 361 — the rule gives 73 on `skew` and 128 on
// config 3.
pepp_status_t prepare_sell_long(pepp_spmv_plan_t* p, int64_t* nnz_long) {
    *nnz_long = 0;
    int64_t cap = kSellCapMin;
    {
        int occ = 0;
        const void* fn = p->vt == PEPP_VALUE_F32 ? (const void*)pepp::k::sell_kernel<kBlock, true, false, float>
                                                 : (const void*)pepp::k::sell_kernel<kBlock, true, false, double>;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, kBlock, 0) != cudaSuccess || occ < 1) occ = 1;
        (void)cudaGetLastError();
        const int64_t warps = (int64_t)std::max(1, p->sm_count - p->reserve_sms) * occ * (kBlock / 32);
        const int64_t nchunks = (p->nrows + 31) / 32;
        const int64_t share = (p->info.nnz / 32 + kChunkCost * nchunks + warps - 1) / warps;
        const int64_t rel = (int64_t)std::ceil(8.0 * p->info.mean_row);
        cap = std::max<int64_t>(cap, std::min(share, rel));
    }
#ifdef PEPP_EXP_SELL_CAP   // experiments only: a fixed cap, set at build time (PEPP_NVCC_EXTRA=-DPEPP_EXP_SELL_CAP=n)
    cap = std::max(1, PEPP_EXP_SELL_CAP);
#endif
    p->sell_cap = (int)std::min<int64_t>(cap, INT32_MAX);
    if (p->info.max_row <= cap) return PEPP_OK;
    const int64_t n = p->nrows;
    std::vector<int> rp(n + 1);
    PEPP_CUDA_TRY(cudaMemcpy(rp.data(), p->d_rp, sizeof(int) * (n + 1), cudaMemcpyDeviceToHost));
    std::vector<int4> seg;
    std::vector<int2> lrow;
    std::vector<int> mid;
    const int64_t mid_max = kSellMidMax;
    for (int64_t r = 0; r < n; ++r) {
        const int b = rp[r], e = rp[r + 1];
        if (e - b <= cap) continue;
        *nnz_long += e - b;
        if (e - b <= mid_max) { mid.push_back((int)r); continue; }
        const int li = (int)lrow.size();
        lrow.push_back(make_int2((int)seg.size(), 0));
        for (int k = b; k < e; k += pepp::k::kSellLongSeg)
            seg.push_back(make_int4((int)r, k, std::min(e, k + pepp::k::kSellLongSeg), li));
        lrow.back().y = (int)seg.size() - lrow.back().x;
    }
    pepp_status_t s;
    if (!mid.empty()) {
        if ((s = dalloc(p, &p->d_sell_mid, (int64_t)mid.size()))) return s;
        PEPP_CUDA_TRY(cudaMemcpy(p->d_sell_mid, mid.data(), sizeof(int) * mid.size(), cudaMemcpyHostToDevice));
        p->nsell_mid = (int)mid.size();
    }
    if (seg.empty()) return PEPP_OK;
    if ((s = dalloc(p, &p->d_sell_seg, (int64_t)seg.size()))) return s;
    if ((s = dalloc(p, &p->d_sell_lrow, (int64_t)lrow.size()))) return s;
    if ((s = dalloc(p, &p->d_sell_cnt, (int64_t)lrow.size()))) return s;
    if ((s = dalloc_bytes(p, &p->d_sell_part, 8 * (int64_t)seg.size()))) return s;
    PEPP_CUDA_TRY(cudaMemcpy(p->d_sell_seg, seg.data(), sizeof(int4) * seg.size(), cudaMemcpyHostToDevice));
    PEPP_CUDA_TRY(cudaMemcpy(p->d_sell_lrow, lrow.data(), sizeof(int2) * lrow.size(), cudaMemcpyHostToDevice));
    PEPP_CUDA_TRY(cudaMemset(p->d_sell_cnt, 0, sizeof(unsigned int) * lrow.size()));
    p->nsell_seg = (int)seg.size();
    p->nsell_long = (int)lrow.size();
    return PEPP_OK;
}

pepp_status_t sell_stencil_list(pepp_spmv_plan_t* p);

// Bytes one SELL call moves from / to HBM with the layout as stored — the
// physical roofline numerator (bench.py `roofline`): per chunk of the
// general walk its descriptor (chunk_ptr 8 B + chunk_len 4 B, + a 4 B list
// entry when walked through a list), its values (slots x value size, none
// for a pattern-table chunk), its index stream (stencil: one 4 B offset per
// slot for the whole chunk; 16-bit deltas: 2 B per slot; else 4 B per slot),
// row lengths of masked chunks (4 B per row) and the permutation (4 B per
// row, σ > 1); stencil-list chunks: values + one 8 B list entry; hybrid rows
// (mid / long kernels): their CSR entries (value + 4 B column), 2 row
// pointers and a 4 B row id or a 16 B segment + 2 x 8 B partial; plus x
// read once (ncols) and y written once (nrows). Padding slots count: they
// are streamed.
pepp_status_t sell_layout_bytes(pepp_spmv_plan_t* p) {
    using pepp::k::kSellLenMask;
    const int nc = p->nchunks;
    const int64_t es = (int64_t)p->esz;
    std::vector<int> clen(nc);
    if (nc) PEPP_CUDA_TRY(cudaMemcpy(clen.data(), p->d_chunk_len, sizeof(int) * nc, cudaMemcpyDeviceToHost));
    std::vector<uint8_t> in_list(nc, 0);
    if (p->d_stlist && p->nstc) {
        std::vector<int2> l(p->nstc);
        PEPP_CUDA_TRY(cudaMemcpy(l.data(), p->d_stlist, sizeof(int2) * p->nstc, cudaMemcpyDeviceToHost));
        for (const int2& e : l) in_list[e.x & ((1 << 26) - 1)] = 1;
    }
    const bool lists = p->d_genlist != nullptr;   // general chunks reached through a 4 B list entry
    int64_t b = 0;
    for (int c = 0; c < nc; ++c) {
        const int d = clen[c];
        const int64_t len = d & kSellLenMask, slots = 32 * len;
        if (in_list[c]) { b += slots * es + 8; continue; }
        if (d & pepp::k::kSellPattern) { b += 4; continue; }   // patlist entry; offsets and values are kernel parameters
        b += 12 + (lists ? 4 : 0) + slots * es;
        if (d & pepp::k::kSellStencil) b += 4 * len;
        else if (d & pepp::k::kSellCol16) b += 2 * slots;
        else b += 4 * slots;
        if (d & pepp::k::kSellMasked) b += 4 * 32;
    }
    if (p->d_perm) b += 4 * p->nrows;
    b += 16 * (int64_t)p->ptl.ntiles - 4 * p->ptl.chunks;   // tiled pattern chunks: one 16 B tile entry per tile
    b += 16 * (int64_t)p->stl.ntiles - 8 * p->stl.chunks;   // tiled stencil-list chunks: likewise
    b += p->sell_long_nnz * (es + 4) + (int64_t)p->nsell_mid * (4 + 8) + (int64_t)p->nsell_long * 8 +
         (int64_t)p->nsell_seg * (16 + 16);
    b += p->ncols * es + p->nrows * es;
    p->sell_bytes = b;
    return PEPP_OK;
}

pepp_status_t prepare_sell(pepp_spmv_plan_t* p, cudaStream_t st) {
    const int n = (int)p->nrows;
    p->nchunks = (n + 31) / 32;
    if (n == 0) return PEPP_OK;
    pepp_status_t s;
    if ((s = dalloc(p, &p->d_chunk_len, p->nchunks))) return s;
    if ((s = dalloc(p, &p->d_rowlen, n))) return s;
    if ((s = dalloc(p, &p->d_chunk_ptr, (int64_t)p->nchunks + 1))) return s;
    const int tb = 256, gb = (n + tb - 1) / tb;
    int64_t nnz_long = 0;
    if ((s = prepare_sell_long(p, &nnz_long))) return s;
    p->sell_long_nnz = nnz_long;
    const int cap = p->sell_cap;

    auto fill_ratio = [&](const int* perm, double* fill) -> pepp_status_t {
        pepp::k::sell_lengths_kernel<<<gb, tb, 0, st>>>(n, p->d_rp, perm, cap, p->d_rowlen, p->d_chunk_len);
        PEPP_CUDA_TRY(cudaGetLastError());
        std::vector<int> cl(p->nchunks);
        PEPP_CUDA_TRY(cudaMemcpyAsync(cl.data(), p->d_chunk_len, sizeof(int) * p->nchunks, cudaMemcpyDeviceToHost, st));
        PEPP_CUDA_TRY(cudaStreamSynchronize(st));
        int64_t slots = 0;
        std::vector<int64_t> cp(p->nchunks + 1);
        for (int c = 0; c < p->nchunks; ++c) { cp[c] = slots; slots += (int64_t)(cl[c] & pepp::k::kSellLenMask) * 32; }
        cp[p->nchunks] = slots;
        p->sell_slots = slots;
        *fill = p->nnz - nnz_long > 0 ? (double)slots / (double)(p->nnz - nnz_long) : 1.0;
        PEPP_CUDA_TRY(cudaMemcpyAsync(p->d_chunk_ptr, cp.data(), sizeof(int64_t) * (p->nchunks + 1), cudaMemcpyHostToDevice, st));
        PEPP_CUDA_TRY(cudaStreamSynchronize(st));
        return PEPP_OK;
    };

    double fill = 1.0;
    int sigma = p->opts.sell_sigma;
    if (sigma <= 1) {
        if ((s = fill_ratio(nullptr, &fill))) return s;
        sigma = 1;
        if (p->opts.sell_sigma == 0 && fill > 1.15) sigma = 4096;   // auto: sort when σ=1 pads > 15 %
    }
    if (sigma > 1) {
        // stable radix sort of (window, maxlen - len) keys -> perm
        DevTmp<unsigned long long> keys, keys_out;
        DevTmp<int> rows;
        DevTmp<unsigned char> tmp;
        size_t tmp_cap = 0;
        const int maxlen = (int)p->info.max_row;
        PEPP_CUDA_TRY(keys.alloc(n));
        PEPP_CUDA_TRY(keys_out.alloc(n));
        PEPP_CUDA_TRY(rows.alloc(n));
        if ((s = dalloc(p, &p->d_perm, n))) return s;
        auto sort_for = [&](int sg, double* f) -> pepp_status_t {
            size_t tmp_bytes = 0;
            pepp::k::sell_keys_kernel<<<gb, tb, 0, st>>>(n, p->d_rp, sg, maxlen, cap, keys.p, rows.p);
            PEPP_CUDA_TRY(cudaGetLastError());
            int end_bit = 32;
            while ((1ull << (end_bit - 32)) <= (unsigned long long)((n - 1) / sg) && end_bit < 64) ++end_bit;
            cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, keys.p, keys_out.p, rows.p, p->d_perm, n, 0, end_bit, st);
            if (!tmp.p || tmp_bytes > tmp_cap) {
                if (tmp.p) { cudaFree(tmp.p); tmp.p = nullptr; }
                PEPP_CUDA_TRY(tmp.alloc(tmp_bytes));
                tmp_cap = tmp_bytes;
            }
            PEPP_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp.p, tmp_bytes, keys.p, keys_out.p, rows.p, p->d_perm, n, 0, end_bit, st));
            PEPP_CUDA_TRY(cudaStreamSynchronize(st));
            return fill_ratio(p->d_perm, f);
        };
        if ((s = sort_for(sigma, &fill))) return s;
    }
    p->sell_sigma = sigma;
    if ((s = dalloc(p, &p->d_scol, p->sell_slots + 32))) return s;
    if ((s = dalloc_bytes(p, &p->d_sval, (p->sell_slots + 32) * (int64_t)p->esz))) return s;
    // padding slots are never read (lanes mask by row length), but keep them defined
    PEPP_CUDA_TRY(cudaMemsetAsync(p->d_scol, 0, sizeof(int) * (p->sell_slots + 32), st));
    PEPP_CUDA_TRY(cudaMemsetAsync(p->d_sval, 0, p->esz * (p->sell_slots + 32), st));
    if (p->vt == PEPP_VALUE_F32)
        pepp::k::sell_fill_kernel<float><<<gb, tb, 0, st>>>(n, p->d_rp, p->d_perm, cap, p->d_col, (const float*)p->d_val,
                                                            p->d_chunk_ptr, p->d_scol, (float*)p->d_sval);
    else
        pepp::k::sell_fill_kernel<double><<<gb, tb, 0, st>>>(n, p->d_rp, p->d_perm, cap, p->d_col, (const double*)p->d_val,
                                                             p->d_chunk_ptr, p->d_scol, (double*)p->d_sval);
    PEPP_CUDA_TRY(cudaGetLastError());
    // stencil chunks: one offset per slot for the whole chunk (no column stream)
    {
        if ((s = dalloc(p, &p->d_soff, p->sell_slots / 32 + 8))) return s;
        const int64_t nsb = p->sell_slots / 32 + 8;   // per-chunk slot tables are indexed by chunk_ptr / 32
        DevTmp<double> d_sconst;                      // 8-byte slots hold either value type
        DevTmp<unsigned char> d_cflag;
        if (p->opts.compress_values) {
            PEPP_CUDA_TRY(d_sconst.alloc(nsb));
            PEPP_CUDA_TRY(d_cflag.alloc(p->nchunks));
            PEPP_CUDA_TRY(cudaMemsetAsync(d_cflag.p, 0, p->nchunks, st));
        }
        DevTmp<unsigned long long> d_nst;
        PEPP_CUDA_TRY(d_nst.alloc(2));
        PEPP_CUDA_TRY(cudaMemsetAsync(d_nst.p, 0, 2 * sizeof(unsigned long long), st));
        const int wb = 256, wg = (int)(((int64_t)p->nchunks * 32 + wb - 1) / wb);
        if (p->vt == PEPP_VALUE_F32)
            pepp::k::sell_stencil_kernel<float><<<wg, wb, 0, st>>>(n, p->nchunks, p->d_chunk_ptr, p->d_chunk_len, p->d_perm,
                p->d_scol, p->d_soff, d_nst.p, (const float*)p->d_sval, (float*)d_sconst.p, d_cflag.p, d_nst.p + 1);
        else
            pepp::k::sell_stencil_kernel<double><<<wg, wb, 0, st>>>(n, p->nchunks, p->d_chunk_ptr, p->d_chunk_len, p->d_perm,
                p->d_scol, p->d_soff, d_nst.p, (const double*)p->d_sval, d_sconst.p, d_cflag.p, d_nst.p + 1);
        PEPP_CUDA_TRY(cudaGetLastError());
        unsigned long long nst[2] = {0, 0};
        PEPP_CUDA_TRY(cudaMemcpyAsync(nst, d_nst.p, sizeof(nst), cudaMemcpyDeviceToHost, st));
        PEPP_CUDA_TRY(cudaStreamSynchronize(st));
        p->sell_stencil_chunks = (int64_t)nst[0];
        if (nst[1] > 0) {
            if (p->vt == PEPP_VALUE_F32) s = sell_patterns<float>(p, nsb, d_sconst.p, d_cflag.p, &p->pat32);
            else s = sell_patterns<double>(p, nsb, d_sconst.p, d_cflag.p, &p->pat64);
            if (s) return s;
        }
    }
    // 16-bit column deltas where a whole chunk allows them (banded / stencil
    // structure): 2 instead of 4 bytes of index per stored slot
    {
        if ((s = dalloc(p, &p->d_scol16, p->sell_slots + 32))) return s;
        PEPP_CUDA_TRY(cudaMemsetAsync(p->d_scol16, 0, sizeof(int16_t) * (p->sell_slots + 32), st));
        DevTmp<unsigned long long> d_n16;
        PEPP_CUDA_TRY(d_n16.alloc(1));
        PEPP_CUDA_TRY(cudaMemsetAsync(d_n16.p, 0, sizeof(unsigned long long), st));
        const int wb = 256, wg = (int)(((int64_t)p->nchunks * 32 + wb - 1) / wb);
        pepp::k::sell_col16_kernel<<<wg, wb, 0, st>>>(n, p->nchunks, p->d_chunk_ptr, p->d_chunk_len, p->d_rowlen,
                                                       p->d_perm, p->d_scol, p->d_scol16, d_n16.p);
        PEPP_CUDA_TRY(cudaGetLastError());
        unsigned long long n16 = 0;
        PEPP_CUDA_TRY(cudaMemcpyAsync(&n16, d_n16.p, sizeof(n16), cudaMemcpyDeviceToHost, st));
        PEPP_CUDA_TRY(cudaStreamSynchronize(st));
        p->sell_col16_chunks = (int64_t)n16;
        if (n16 == 0) { cudaFree(p->d_scol16); p->d_scol16 = nullptr; p->dev_bytes -= (int64_t)sizeof(int16_t) * (p->sell_slots + 32); }
    }
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    if ((s = sell_stencil_list(p))) return s;
    if ((s = sell_layout_bytes(p))) return s;
    p->sell_cpw = sigma > 1 ? std::max(1, sigma / 32) : 1;
    p->info.sell_sigma = sigma;
    p->info.sell_col16_frac = p->nchunks ? (double)p->sell_col16_chunks / (double)p->nchunks : 0.0;
    p->info.sell_stencil_frac = p->nchunks ? (double)p->sell_stencil_chunks / (double)p->nchunks : 0.0;
    p->info.sell_constval_frac = p->nchunks ? (double)p->sell_const_chunks / (double)p->nchunks : 0.0;
    p->info.sell_ptile_frac = p->nchunks ? (double)(p->ptl.chunks + p->stl.chunks) / (double)p->nchunks : 0.0;
    p->info.sell_tile_multiline = p->ptl.lines;
    p->info.sell_fill = fill;
    p->info.sell_long_rows = p->nsell_long + p->nsell_mid;
    p->info.sell_cap = p->sell_cap == INT32_MAX ? 0 : p->sell_cap;
    return PEPP_OK;
}

// Stencil list for σ = 1 plans whose stencil chunks stream their values (no
// pattern table): unmasked stencil chunks of <= 16 slots, grouped by offset
// set (<= kSellMaxStencils sets; chunks of further sets stay general), for
// sell_slist_kernel; every other chunk goes to the genlist for sell_kernel.
pepp_status_t sell_stencil_list(pepp_spmv_plan_t* p) {
    using pepp::k::kSellLenMask;
    const int nc = p->nchunks;
    if (p->d_perm || p->d_patlist || p->sell_stencil_chunks == 0 || nc <= 0) return PEPP_OK;
    // measured on config 4 (3 alternating repeats each): fp32 424 -> 361 µs
    // (the issue-limited general walk loses its per-chunk instructions,
    // tools/gpu_slist2.sh), 349 µs with the genlist walk concurrent; fp64
    // 593-596 -> 578.5 µs with the concurrent genlist walk (tools/gpu_slist5.sh;
    // 582.5 with it sequential)
    if (p->vt == PEPP_VALUE_F64 && !kSlistF64) return PEPP_OK;
    const int64_t nsb = p->sell_slots / 32 + 8;
    std::vector<int> clen(nc), soff(nsb);
    std::vector<int64_t> cp(nc + 1);
    PEPP_CUDA_TRY(cudaMemcpy(clen.data(), p->d_chunk_len, sizeof(int) * nc, cudaMemcpyDeviceToHost));
    PEPP_CUDA_TRY(cudaMemcpy(cp.data(), p->d_chunk_ptr, sizeof(int64_t) * (nc + 1), cudaMemcpyDeviceToHost));
    PEPP_CUDA_TRY(cudaMemcpy(soff.data(), p->d_soff, sizeof(int) * nsb, cudaMemcpyDeviceToHost));
    pepp::k::SellStencils tab{};
    int nset = 0;
    std::vector<int2> lst;
    std::vector<int> gen;
    lst.reserve(nc);
    for (int c = 0; c < nc; ++c) {
        const int d = clen[c], len = d & kSellLenMask;
        int pid = -1;
        if ((d & pepp::k::kSellStencil) && !(d & pepp::k::kSellMasked) && len >= 1 && len <= pepp::k::kSellMaxStencilLen &&
            c < (1 << 26) && (cp[c] >> 5) <= INT32_MAX) {
            const int64_t sb = cp[c] >> 5;
            for (int q = 0; q < nset && pid < 0; ++q) {
                bool same = tab.len[q] == len;
                for (int j = 0; same && j < len; ++j) same = tab.off[q][j] == soff[sb + j];
                if (same) pid = q;
            }
            if (pid < 0 && nset < pepp::k::kSellMaxStencils) {
                pid = nset++;
                tab.len[pid] = len;
                for (int j = 0; j < len; ++j) tab.off[pid][j] = soff[sb + j];
            }
        }
        if (pid >= 0) lst.push_back(make_int2(c | (pid << 26), (int)(cp[c] >> 5)));
        else gen.push_back(c);
    }
    // worth it only when the list carries most chunks: otherwise the genlist
    // walk (the PAT instance, no pairing) would take the bulk (measured on
    // banded b = 4, 9-slot chunks: 1833 -> 2065 µs at 10^8 rows)
    if (lst.empty() || 2 * (int64_t)lst.size() < (int64_t)nc) return PEPP_OK;
    std::stable_sort(lst.begin(), lst.end(), [](const int2& a, const int2& b) { return (a.x >> 26) < (b.x >> 26); });
    pepp_status_t s;
    if ((s = dalloc(p, &p->d_stlist, (int64_t)lst.size()))) return s;
    if ((s = dalloc(p, &p->d_genlist, (int64_t)gen.size()))) return s;
    PEPP_CUDA_TRY(cudaMemcpy(p->d_stlist, lst.data(), sizeof(int2) * lst.size(), cudaMemcpyHostToDevice));
    if (!gen.empty()) PEPP_CUDA_TRY(cudaMemcpy(p->d_genlist, gen.data(), sizeof(int) * gen.size(), cudaMemcpyHostToDevice));
    p->nstc = (int)lst.size();
    p->ngen = (int)gen.size();
    p->stab = tab;
    // stencil tiles over the list (the untiled entries -> d_strest)
    if (kStencilTiles & (p->vt == PEPP_VALUE_F32 ? 1 : 2)) {
        std::vector<int4> ents(lst.size());
        for (size_t i = 0; i < lst.size(); ++i)
            ents[i] = make_int4(lst[i].x & ((1 << 26) - 1), lst[i].x >> 26, lst[i].y, 0);
        std::vector<size_t> rest;
        int offs[pepp::k::kTileMaxSets][pepp::k::kTileMaxLen] = {{0}};
        for (int q = 0; q < nset; ++q)
            for (int j = 0; j < tab.len[q]; ++j) offs[q][j] = tab.off[q][j];
        pepp_status_t st2 = p->vt == PEPP_VALUE_F32
            ? sell_build_tiles<float>(p, nset, tab.len, offs, ents, true, &p->stl, &rest)
            : sell_build_tiles<double>(p, nset, tab.len, offs, ents, true, &p->stl, &rest);
        if (st2) return st2;
        if (p->stl.ntiles && !rest.empty()) {
            std::sort(rest.begin(), rest.end());
            std::vector<int2> r(rest.size());
            for (size_t i = 0; i < rest.size(); ++i) r[i] = lst[rest[i]];
            if ((s = dalloc(p, &p->d_strest, (int64_t)r.size()))) return s;
            PEPP_CUDA_TRY(cudaMemcpy(p->d_strest, r.data(), sizeof(int2) * r.size(), cudaMemcpyHostToDevice));
            p->nstrest = (int)r.size();
        }
        if (p->stl.ntiles && (p->nstrest || p->ngen) && (s = ensure_side_stream(p))) return s;
    }
    if (p->ngen > 0 && kSlistConcurrent && !p->gside) {
        PEPP_CUDA_TRY(cudaStreamCreateWithFlags(&p->gside, cudaStreamNonBlocking));
        PEPP_CUDA_TRY(cudaEventCreateWithFlags(&p->ev_gfork, cudaEventDisableTiming));
        PEPP_CUDA_TRY(cudaEventCreateWithFlags(&p->ev_gjoin, cudaEventDisableTiming));
    }
    int occ = 0;
    int lmax = 0;
    for (int q = 0; q < nset; ++q) lmax = std::max(lmax, tab.len[q]);
    p->slist_long = lmax > 8;
    const bool lg = p->slist_long;
    const void* fn = p->vt == PEPP_VALUE_F32
        ? (lg ? (const void*)pepp::k::sell_slist_kernel<kBlock, pepp::k::sell_slist_u<float, 16>(), 16, float>
              : (const void*)pepp::k::sell_slist_kernel<kBlock, pepp::k::sell_slist_u<float>(), 8, float>)
        : (lg ? (const void*)pepp::k::sell_slist_kernel<kBlock, pepp::k::sell_slist_u<double, 16>(), 16, double>
              : (const void*)pepp::k::sell_slist_kernel<kBlock, pepp::k::sell_slist_u<double>(), 8, double>);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, kBlock, 0) != cudaSuccess || occ < 1) occ = 1;
    (void)cudaGetLastError();
    const int64_t need = ((int64_t)p->nstc + kBlock / 32 - 1) / (kBlock / 32);
    p->grid_slist = (int)std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)std::max(1, p->sm_count - p->reserve_sms) * occ));
    return PEPP_OK;
}

// ---------------------------------------------------------------- panel prep
// The column-panel layout (variant PEPP_V_PANEL) pays only where x is far
// larger than L2 and the rows reach across it (random columns): x > 96 MB
// and a mean row span (last - first column) above half a panel. One layout
// per panel width 2^lg (x panel of 32 MB and, when memory is modest, 64 MB):
// a stable radix sort of the entries by panel (CSR order kept within a
// panel), the (row, panel) pairs by head flags (cub select), their pair
// ranges per panel by binary search.
#ifndef PEPP_PANEL_MIN_MB
#define PEPP_PANEL_MIN_MB 96   // checked below it (tools/r2/panel_mid.py, threshold 24 MB): uniform 16/row at 6e6 / 1e7 / 1.2e7 rows
#endif                         // panel[22] 862 / 1347 / 1536 us vs sell[1] 413 / 860 / 1450 us
constexpr int64_t kPanelMinX = (int64_t)PEPP_PANEL_MIN_MB << 20;

pepp_status_t prepare_panels(pepp_spmv_plan_t* p, cudaStream_t st, std::vector<int>* lgs) {
    lgs->clear();
    const int64_t n = p->nnz, R = p->nrows;
    if (p->ncols * (int64_t)p->esz <= kPanelMinX || n == 0 || R == 0) return PEPP_OK;
    // mean row span
    {
        DevTmp<unsigned long long> d_span;
        PEPP_CUDA_TRY(d_span.alloc(1));
        PEPP_CUDA_TRY(cudaMemsetAsync(d_span.p, 0, sizeof(unsigned long long), st));
        pepp::k::row_span_kernel<<<std::min<int64_t>((R + 255) / 256, (int64_t)p->sm_count * 8), 256, 0, st>>>(
            R, p->d_rp, p->d_col, d_span.p);
        PEPP_CUDA_TRY(cudaGetLastError());
        unsigned long long span = 0;
        PEPP_CUDA_TRY(cudaMemcpyAsync(&span, d_span.p, sizeof(span), cudaMemcpyDeviceToHost, st));
        PEPP_CUDA_TRY(cudaStreamSynchronize(st));
#ifndef PEPP_PANEL_LG0
#define PEPP_PANEL_LG0 22   // experiments: log2 entries of the first fp64 panel width (32 MB of x)
#endif
        const int lg0 = p->esz == 8 ? PEPP_PANEL_LG0 : PEPP_PANEL_LG0 + 1;   // 32 MB of x per panel
        if ((double)span / (double)R < (double)(1ll << (lg0 - 1))) return PEPP_OK;
        lgs->push_back(lg0);
        if ((double)n * 2.0 * (4.0 + (double)p->esz) <= 48e9) lgs->push_back(lg0 + 1);   // and 64 MB, memory permitting
    }
    std::vector<int> ok;
    for (int lg : *lgs) {
        const int npanels = (int)((p->ncols + (1ll << lg) - 1) >> lg);
        if (npanels < 2 || npanels > 255) continue;
        p->panels.emplace_back();   // owned by the plan from here on: freed with it on any error path
        PanelLayout& L = p->panels.back();
        L.lg = lg;
        L.npanels = npanels;
        pepp_status_t s;
        DevTmp<unsigned char> key, skey, head;
        DevTmp<int> idx, sidx, row_of, prow_full, starts;
        DevTmp<int> nsel;
        DevTmp<unsigned char> tmp;
        PEPP_CUDA_TRY(key.alloc(n));
        PEPP_CUDA_TRY(skey.alloc(n));
        PEPP_CUDA_TRY(idx.alloc(n));
        PEPP_CUDA_TRY(sidx.alloc(n));
        PEPP_CUDA_TRY(row_of.alloc(n));
        const int gb = (int)std::min<int64_t>((R + 255) / 256, (int64_t)p->sm_count * 16);
        pepp::k::panel_keys_kernel<<<gb, 256, 0, st>>>(R, p->d_rp, p->d_col, lg, p->pad, key.p, row_of.p, idx.p);
        PEPP_CUDA_TRY(cudaGetLastError());
        int end_bit = 1;
        while ((1 << end_bit) < npanels) ++end_bit;
        size_t tb = 0;
        PEPP_CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, key.p, skey.p, idx.p, sidx.p, (int)n, 0, end_bit, st));
        PEPP_CUDA_TRY(tmp.alloc(tb));
        PEPP_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp.p, tb, key.p, skey.p, idx.p, sidx.p, (int)n, 0, end_bit, st));
        { DevTmp<unsigned char> k2; std::swap(k2.p, key.p); DevTmp<int> i2; std::swap(i2.p, idx.p); }   // free early
        if ((s = dalloc(p, &L.d_pcol, n))) return s;
        if ((s = dalloc_bytes(p, &L.d_pval, n * (int64_t)p->esz))) return s;
        PEPP_CUDA_TRY(prow_full.alloc(n));
        PEPP_CUDA_TRY(head.alloc(n));
        const int gn = (int)std::min<int64_t>((n + 255) / 256, (int64_t)p->sm_count * 32);
        if (p->vt == PEPP_VALUE_F32)
            pepp::k::panel_gather_kernel<float><<<gn, 256, 0, st>>>(n, p->pad, sidx.p, p->d_col, (const float*)p->d_val,
                                                                   row_of.p, skey.p, L.d_pcol, (float*)L.d_pval, prow_full.p, head.p);
        else
            pepp::k::panel_gather_kernel<double><<<gn, 256, 0, st>>>(n, p->pad, sidx.p, p->d_col, (const double*)p->d_val,
                                                                    row_of.p, skey.p, L.d_pcol, (double*)L.d_pval, prow_full.p, head.p);
        PEPP_CUDA_TRY(cudaGetLastError());
        PEPP_CUDA_TRY(starts.alloc(n + 1));
        PEPP_CUDA_TRY(nsel.alloc(1));
        thrust::counting_iterator<int> it(0);
        size_t tb2 = 0;
        PEPP_CUDA_TRY(cub::DeviceSelect::Flagged(nullptr, tb2, it, head.p, starts.p, nsel.p, (int)n, st));
        DevTmp<unsigned char> tmp2;
        PEPP_CUDA_TRY(tmp2.alloc(tb2));
        PEPP_CUDA_TRY(cub::DeviceSelect::Flagged(tmp2.p, tb2, it, head.p, starts.p, nsel.p, (int)n, st));
        int np = 0;
        PEPP_CUDA_TRY(cudaMemcpyAsync(&np, nsel.p, sizeof(int), cudaMemcpyDeviceToHost, st));
        PEPP_CUDA_TRY(cudaStreamSynchronize(st));
        L.npairs = np;
        if ((s = dalloc(p, &L.d_prow, np))) return s;
        if ((s = dalloc(p, &L.d_pstart, (int64_t)np + 1))) return s;
        const int nn = (int)n;
        PEPP_CUDA_TRY(cudaMemcpyAsync(L.d_pstart, starts.p, sizeof(int) * np, cudaMemcpyDeviceToDevice, st));
        PEPP_CUDA_TRY(cudaMemcpyAsync(L.d_pstart + np, &nn, sizeof(int), cudaMemcpyHostToDevice, st));
        pepp::k::panel_pairs_kernel<<<(int)std::min<int64_t>(((int64_t)np + 255) / 256, (int64_t)p->sm_count * 32), 256, 0, st>>>(
            np, starts.p, prow_full.p, L.d_prow);
        PEPP_CUDA_TRY(cudaGetLastError());
        // pair ranges per panel
        DevTmp<int64_t> zoff;
        DevTmp<int> poff;
        PEPP_CUDA_TRY(zoff.alloc(npanels + 1));
        PEPP_CUDA_TRY(poff.alloc(npanels + 1));
        std::vector<int64_t> hz(npanels + 1, -1);
        PEPP_CUDA_TRY(cudaMemcpyAsync(zoff.p, hz.data(), sizeof(int64_t) * (npanels + 1), cudaMemcpyHostToDevice, st));
        pepp::k::panel_bounds_kernel<<<gn, 256, 0, st>>>(n, skey.p, zoff.p);
        PEPP_CUDA_TRY(cudaGetLastError());
        PEPP_CUDA_TRY(cudaMemcpyAsync(hz.data(), zoff.p, sizeof(int64_t) * (npanels + 1), cudaMemcpyDeviceToHost, st));
        PEPP_CUDA_TRY(cudaStreamSynchronize(st));
        hz[npanels] = n;
        for (int k = npanels - 1; k >= 0; --k) if (hz[k] < 0) hz[k] = hz[k + 1];   // empty panels
        PEPP_CUDA_TRY(cudaMemcpyAsync(zoff.p, hz.data(), sizeof(int64_t) * (npanels + 1), cudaMemcpyHostToDevice, st));
        pepp::k::panel_pair_offsets_kernel<<<(npanels + 1 + 255) / 256, 256, 0, st>>>(npanels, zoff.p, L.d_pstart, np, poff.p);
        PEPP_CUDA_TRY(cudaGetLastError());
        L.poff.resize(npanels + 1);
        PEPP_CUDA_TRY(cudaMemcpyAsync(L.poff.data(), poff.p, sizeof(int) * (npanels + 1), cudaMemcpyDeviceToHost, st));
        PEPP_CUDA_TRY(cudaStreamSynchronize(st));
        ok.push_back(lg);
    }
    *lgs = ok;
    return PEPP_OK;
}

// ---------------------------------------------------------------- merge prep
// Runs of >= kLongRun consecutive tiles that carry into the same row (the row
// open at a tile's end is tile_coord[t+1].x, fixed by the structure).
pepp_status_t long_runs(pepp_spmv_plan_t* p, const int2* d_tile, int ntiles, int4** out, int* nout) {
    *nout = 0;
    if (ntiles <= 0) return PEPP_OK;
    std::vector<int2> tc(ntiles + 1);
    PEPP_CUDA_TRY(cudaMemcpy(tc.data(), d_tile, sizeof(int2) * (ntiles + 1), cudaMemcpyDeviceToHost));
    std::vector<int4> runs;
    for (int t = 0; t < ntiles;) {
        const int row = tc[t + 1].x;
        int u = t + 1;
        while (u < ntiles && tc[u + 1].x == row) ++u;
        if (row < p->nrows && u - t >= pepp::k::kLongRun) runs.push_back(make_int4(t, u - t, row, 0));
        t = u;
    }
    if (runs.empty()) return PEPP_OK;
    pepp_status_t s;
    if ((s = dalloc(p, out, (int64_t)runs.size()))) return s;
    PEPP_CUDA_TRY(cudaMemcpy(*out, runs.data(), sizeof(int4) * runs.size(), cudaMemcpyHostToDevice));
    *nout = (int)runs.size();
    return PEPP_OK;
}

pepp_status_t prepare_merge(pepp_spmv_plan_t* p, cudaStream_t st) {
    const int64_t total = p->nrows + p->nnz;
    p->ntiles = (int)((total + kMergeTile - 1) / kMergeTile);
    pepp_status_t s;
    if ((s = dalloc(p, &p->d_tile, (int64_t)p->ntiles + 1))) return s;
    if ((s = dalloc(p, &p->d_carry_row, std::max(p->ntiles, 1)))) return s;
    if ((s = dalloc_bytes(p, &p->d_carry_val, 8 * (int64_t)std::max(p->ntiles, 1)))) return s;
    const int tb = 256;
    pepp::k::merge_tile_search_kernel<<<(p->ntiles + 1 + tb - 1) / tb, tb, 0, st>>>(
        (int)p->nrows, p->nnz, p->d_rp, kMergeTile, p->ntiles, p->d_tile);
    PEPP_CUDA_TRY(cudaGetLastError());
    p->ntiles_w = (int)((total + kMergeWarpTile - 1) / kMergeWarpTile);
    if ((s = dalloc(p, &p->d_tile_w, (int64_t)p->ntiles_w + 1))) return s;
    if ((s = dalloc(p, &p->d_carry_row_w, std::max(p->ntiles_w, 1)))) return s;
    if ((s = dalloc_bytes(p, &p->d_carry_val_w, 8 * (int64_t)std::max(p->ntiles_w, 1)))) return s;
    pepp::k::merge_tile_search_kernel<<<(p->ntiles_w + 1 + tb - 1) / tb, tb, 0, st>>>(
        (int)p->nrows, p->nnz, p->d_rp, kMergeWarpTile, p->ntiles_w, p->d_tile_w);
    PEPP_CUDA_TRY(cudaGetLastError());
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    if ((s = long_runs(p, p->d_tile, p->ntiles, &p->d_longruns, &p->nlongruns))) return s;
    if ((s = long_runs(p, p->d_tile_w, p->ntiles_w, &p->d_longruns_w, &p->nlongruns_w))) return s;
    return PEPP_OK;
}

// ---------------------------------------------------------------- CSR-stream prep
template <typename T>
auto stream_kernel() { return pepp::k::csr_stream_tma_kernel<kStreamBlock, kStreamStages, kStreamNB, kStreamRMAX, kStreamVecMinLen, T>; }
template <typename T>
constexpr size_t stream_smem() { return sizeof(pepp::k::StreamStage<kStreamNB, kStreamRMAX, T>) * kStreamStages; }

template <typename T>
pepp_status_t stream_occupancy(int* occ) {
    PEPP_CUDA_TRY(cudaFuncSetAttribute(stream_kernel<T>(), cudaFuncAttributeMaxDynamicSharedMemorySize, (int)stream_smem<T>()));
    PEPP_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, stream_kernel<T>(), kStreamBlock, stream_smem<T>()));
    return PEPP_OK;
}

pepp_status_t prepare_stream(pepp_spmv_plan_t* p, cudaStream_t st) {
    const int64_t R = p->nrows;
    if (R == 0) return PEPP_OK;
    std::vector<int> rp(R + 1);
    PEPP_CUDA_TRY(cudaMemcpyAsync(rp.data(), p->d_rp, sizeof(int) * (R + 1), cudaMemcpyDeviceToHost, st));
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    std::vector<int4> items, longrows;
    items.reserve((size_t)(p->nnz / kStreamNB + R / kStreamRMAX + 16));
    int piece = 0;
    int64_t r = 0;
    while (r < R) {
        const int len = rp[r + 1] - rp[r];
        if (len > kStreamNB) {   // long row -> pieces of kStreamNB nonzeros
            const int first_piece = piece;
            for (int k = rp[r]; k < rp[r + 1]; k += kStreamNB, ++piece)
                items.push_back(make_int4((int)r, -(piece + 1), k, std::min(k + kStreamNB, rp[r + 1])));
            longrows.push_back(make_int4((int)r, first_piece, piece, 0));
            ++r;
            continue;
        }
        const int64_t r0 = r;
        const int k0 = rp[r];
        int maxlen = 0;
        while (r < R && r - r0 < kStreamRMAX && rp[r + 1] - k0 <= kStreamNB) {
            maxlen = std::max(maxlen, rp[r + 1] - rp[r]);
            ++r;
        }
        const int flag = maxlen > kStreamVecMinLen ? pepp::k::kStreamVecFlag : 0;
        items.push_back(make_int4((int)r0, (int)r | flag, k0, rp[r]));
    }
    p->nitems = (int)items.size();
    p->nlong = (int)longrows.size();
    pepp_status_t s;
    if ((s = dalloc(p, &p->d_items, p->nitems))) return s;
    PEPP_CUDA_TRY(cudaMemcpyAsync(p->d_items, items.data(), sizeof(int4) * items.size(), cudaMemcpyHostToDevice, st));
    if (p->nlong) {
        if ((s = dalloc(p, &p->d_longrows, p->nlong))) return s;
        if ((s = dalloc_bytes(p, &p->d_stream_carry, 8 * (int64_t)piece))) return s;
        PEPP_CUDA_TRY(cudaMemcpyAsync(p->d_longrows, longrows.data(), sizeof(int4) * longrows.size(), cudaMemcpyHostToDevice, st));
    }
    int occ = 0;
    if ((s = p->vt == PEPP_VALUE_F32 ? stream_occupancy<float>(&occ) : stream_occupancy<double>(&occ))) return s;
    if (occ < 1) return PEPP_E_UNSUPPORTED;
    p->grid_stream = (int)std::min<int64_t>((int64_t)p->sm_count * occ, p->nitems);
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    return PEPP_OK;
}

// ---------------------------------------------------------------- launches
template <int TPR, typename T>
void launch_csr_vector(const pepp_spmv_plan_t* p, const T* x, T* y, cudaStream_t st, int grid) {
    pepp::k::csr_vector_kernel<TPR, kBlock, T><<<grid, kBlock, 0, st>>>((int)p->nrows, p->d_rp, p->d_col,
                                                                        (const T*)p->d_val, x, y);
}

template <typename T> const pepp::k::SellPatterns<T>& sell_pattern_table(const pepp_spmv_plan_t* p);
template <> const pepp::k::SellPatterns<double>& sell_pattern_table<double>(const pepp_spmv_plan_t* p) { return p->pat64; }
template <> const pepp::k::SellPatterns<float>& sell_pattern_table<float>(const pepp_spmv_plan_t* p) { return p->pat32; }

// The walker warps are a handful per SM: they take the chunks outside the
// tiles only when those are few next to the tiled ones (grid edges). A plan
// whose tiles are a small part (e.g. a few constant-stencil regions in an
// otherwise general matrix) walks the rest with the full-grid SELL kernel on
// the side stream — with the walkers, 524 K general chunks of a 9-point
// stencil beside 250 tiled ones took 34.8 ms instead of ~0.3 ms.
#ifndef PEPP_WALK_RATIO
#define PEPP_WALK_RATIO 16   // walkers when (chunks outside the tiles) x 16 <= tiled chunks,
#endif                       // or at most 8 of them per walker warp
template <bool VALS>
bool walkers_suffice(const pepp_spmv_plan_t* p, const TileLayout& L) {
    const int64_t walkers = (int64_t)tile_walkers<VALS>() * L.grid;
    return (int64_t)p->ngen * PEPP_WALK_RATIO <= L.chunks || (int64_t)p->ngen <= 8 * walkers;
}

// the side stream of a tile call: forked after the work already on st
pepp_status_t side_fork(pepp_spmv_plan_t* p, cudaStream_t st, cudaStream_t* gs) {
    *gs = p->gside && PEPP_EXP_TILE_SIDE == 0 ? p->gside : st;
    if (*gs != st && (cudaEventRecord(p->ev_gfork, st) != cudaSuccess || cudaStreamWaitEvent(*gs, p->ev_gfork, 0) != cudaSuccess))
        return PEPP_E_CUDA;
    return PEPP_OK;
}
pepp_status_t side_join(pepp_spmv_plan_t* p, cudaStream_t st) {
    if (p->gside && PEPP_EXP_TILE_SIDE == 0 &&
        (cudaEventRecord(p->ev_gjoin, p->gside) != cudaSuccess || cudaStreamWaitEvent(st, p->ev_gjoin, 0) != cudaSuccess))
        return PEPP_E_CUDA;
    return PEPP_OK;
}

// one tile-kernel launch; with `walk`, its walker warps take the genlist
template <bool VALS, typename T>
pepp_status_t tile_launch(pepp_spmv_plan_t* p, const TileLayout& L, bool walk, const T* x, T* y, cudaStream_t st) {
    pepp::k::TileWalk wk;
    if (walk && p->ngen > 0 && PEPP_EXP_TILE_SIDE != 2) {
        wk.nrows = (int)p->nrows;
        wk.ngen = p->ngen;
        wk.chunk_ptr = p->d_chunk_ptr;
        wk.chunk_len = p->d_chunk_len;
        wk.rowlen = p->d_rowlen;
        wk.col = p->d_scol;
        wk.col16 = p->d_scol16;
        wk.soff = p->d_soff;
        wk.genlist = p->d_genlist;
    }
    pepp::k::sell_tile_kernel<tile_block<VALS>(), VALS ? kStileS : kPtileS, VALS, T, tile_walkers<VALS>()>
        <<<L.grid, tile_block<VALS>(), L.smem, st>>>(sell_pattern_table<T>(p), L.tt, L.d_tiles, L.ntiles, L.stage, L.vstage,
                                             (const T*)p->d_sval, x, y, p->ncols, wk);
    return PEPP_OK;
}

template <typename T>
pepp_status_t launch_t(pepp_spmv_plan_t* p, const Candidate& c, const T* x, T* y, cudaStream_t st) {
    if (p->nrows == 0) return PEPP_OK;
    const T* val = (const T*)p->d_val;
    switch (c.variant) {
    case PEPP_V_CSR_VECTOR:
        switch (c.param) {
        case 2: launch_csr_vector<2, T>(p, x, y, st, p->grid_csr[1]); break;
        case 4: launch_csr_vector<4, T>(p, x, y, st, p->grid_csr[2]); break;
        case 8: launch_csr_vector<8, T>(p, x, y, st, p->grid_csr[3]); break;
        case 16: launch_csr_vector<16, T>(p, x, y, st, p->grid_csr[4]); break;
        case 32: launch_csr_vector<32, T>(p, x, y, st, p->grid_csr[5]); break;
        default: return PEPP_E_INVALID;
        }
        break;
    case PEPP_V_MERGE_PATH:
        if (c.param == kMergeWarpParam) {
            if (p->ntiles_w > 0) {
                pepp::k::merge_warp_kernel<kMergeWarpIPT, kMergeWarps, T>
                    <<<(p->ntiles_w + kMergeWarps - 1) / kMergeWarps, kMergeWarps * 32, 0, st>>>(
                        (int)p->nrows, p->ntiles_w, p->d_rp, p->d_col, val, x, y, p->d_tile_w, p->d_carry_row_w,
                        (T*)p->d_carry_val_w);
                pepp::k::merge_fixup_kernel<T><<<(p->ntiles_w + 255) / 256, 256, 0, st>>>(
                    p->ntiles_w, (int)p->nrows, p->d_carry_row_w, (const T*)p->d_carry_val_w, y);
                if (p->nlongruns_w)
                    pepp::k::merge_fixup_long_kernel<T><<<(p->nlongruns_w * 32 + 255) / 256, 256, 0, st>>>(
                        p->nlongruns_w, p->d_longruns_w, (const T*)p->d_carry_val_w, y);
            }
            break;
        }
        if (p->ntiles > 0) {
            pepp::k::merge_spmv_kernel<kMergeBlock, kMergeIPT, T><<<p->ntiles, kMergeBlock, 0, st>>>(
                (int)p->nrows, p->d_rp, p->d_col, val, x, y, p->d_tile, p->d_carry_row, (T*)p->d_carry_val);
            pepp::k::merge_fixup_kernel<T><<<(p->ntiles + 255) / 256, 256, 0, st>>>(
                p->ntiles, (int)p->nrows, p->d_carry_row, (const T*)p->d_carry_val, y);
            if (p->nlongruns)
                pepp::k::merge_fixup_long_kernel<T><<<(p->nlongruns * 32 + 255) / 256, 256, 0, st>>>(
                    p->nlongruns, p->d_longruns, (const T*)p->d_carry_val, y);
        }
        break;
    case PEPP_V_CSR_STREAM:
        if (p->nitems > 0) {
            stream_kernel<T>()<<<p->grid_stream, kStreamBlock, stream_smem<T>(), st>>>(
                p->nitems, p->d_items, p->d_rp, p->d_col, val, x, y, (T*)p->d_stream_carry);
            if (p->nlong)
                pepp::k::csr_stream_fixup_kernel<T><<<(p->nlong * 32 + 255) / 256, 256, 0, st>>>(
                    p->nlong, p->d_longrows, (const T*)p->d_stream_carry, y);
        }
        break;
    case PEPP_V_SELL:
        if (p->d_perm && p->sell_const_chunks)   // σ > 1: pattern chunks inline in the sorted walk
            pepp::k::sell_kernel<kBlock, true, true, T><<<p->grid_sell, kBlock, 0, st>>>(
                (int)p->nrows, p->nchunks, p->d_chunk_ptr, p->d_chunk_len, p->d_rowlen, p->d_perm, p->d_scol,
                p->d_scol16, p->d_soff, sell_pattern_table<T>(p), (const T*)p->d_sval, x, y, p->sell_cpw, p->d_sell_ws,
                nullptr, 0, nullptr);
        else if (p->d_perm)
            pepp::k::sell_kernel<kBlock, true, false, T><<<p->grid_sell, kBlock, 0, st>>>(
                (int)p->nrows, p->nchunks, p->d_chunk_ptr, p->d_chunk_len, p->d_rowlen, p->d_perm, p->d_scol,
                p->d_scol16, p->d_soff, pepp::k::NoPatterns{}, (const T*)p->d_sval, x, y, p->sell_cpw, p->d_sell_ws,
                nullptr, 0, nullptr);
        else if (p->d_patlist && p->ptl.ntiles && ((((uintptr_t)x) | ((uintptr_t)y)) & 15) == 0) {
            // pattern tiles (bulk-copied x ranges); the grid-edge chunks by the
            // tile kernel's walker warps, or — with untiled pattern chunks
            // left (phase A) or no walkers — by the genlist walk beside it
            const bool inwalk = tile_walkers<false>() > 0 && p->npatrest == 0 && walkers_suffice<false>(p, p->ptl);
            pepp_status_t s2 = tile_launch<false, T>(p, p->ptl, inwalk, x, y, st);
            if (s2) return s2;
            if (!inwalk && p->ngen + p->npatrest > 0) {
                cudaStream_t gs;
                if ((s2 = side_fork(p, st, &gs))) return s2;
                pepp::k::sell_kernel<kBlock, false, true, T><<<tile_side_grid(p, p->grid_sell), kBlock, 0, gs>>>(
                    (int)p->nrows, p->ngen, p->d_chunk_ptr, p->d_chunk_len, p->d_rowlen, nullptr,
                    p->d_scol, p->d_scol16, p->d_soff, sell_pattern_table<T>(p), (const T*)p->d_sval, x, y, 1, nullptr,
                    p->d_patrest, p->npatrest, p->d_genlist);
                if ((s2 = side_join(p, st))) return s2;
            }
        } else if (p->d_patlist)   // pattern chunks (value compression): phase A + the rest through genlist
            pepp::k::sell_kernel<kBlock, false, true, T><<<p->grid_sell, kBlock, 0, st>>>(
                (int)p->nrows, p->ngen, p->d_chunk_ptr, p->d_chunk_len, p->d_rowlen, nullptr,
                p->d_scol, p->d_scol16, p->d_soff, sell_pattern_table<T>(p), (const T*)p->d_sval, x, y, 1, nullptr,
                p->d_patlist, p->npatc, p->d_genlist);
        else if (p->d_stlist && p->stl.ntiles && ((((uintptr_t)x) | ((uintptr_t)y)) & 15) == 0) {
            // stencil tiles (bulk-copied x ranges and values); the grid-edge
            // chunks by the walker warps; untiled list entries (and, without
            // walkers, the grid-edge chunks) beside it on the side stream
            const bool inwalk = tile_walkers<true>() > 0 && walkers_suffice<true>(p, p->stl);
            pepp_status_t s2 = tile_launch<true, T>(p, p->stl, inwalk, x, y, st);
            if (s2) return s2;
            if (p->nstrest || (!inwalk && p->ngen > 0)) {
                cudaStream_t gs;
                if ((s2 = side_fork(p, st, &gs))) return s2;
                if (p->nstrest) {
                    if (p->slist_long)
                        pepp::k::sell_slist_kernel<kBlock, pepp::k::sell_slist_u<T, 16>(), 16, T><<<tile_side_grid(p, p->grid_slist), kBlock, 0, gs>>>(
                            p->d_strest, p->nstrest, p->stab, (const T*)p->d_sval, x, y);
                    else
                        pepp::k::sell_slist_kernel<kBlock, pepp::k::sell_slist_u<T>(), 8, T><<<tile_side_grid(p, p->grid_slist), kBlock, 0, gs>>>(
                            p->d_strest, p->nstrest, p->stab, (const T*)p->d_sval, x, y);
                }
                if (!inwalk && p->ngen > 0)
                    pepp::k::sell_kernel<kBlock, false, true, T><<<tile_side_grid(p, p->grid_sell), kBlock, 0, gs>>>(
                        (int)p->nrows, p->ngen, p->d_chunk_ptr, p->d_chunk_len, p->d_rowlen, nullptr,
                        p->d_scol, p->d_scol16, p->d_soff, sell_pattern_table<T>(p), (const T*)p->d_sval, x, y, 1, nullptr,
                        nullptr, 0, p->d_genlist);
                if ((s2 = side_join(p, st))) return s2;
            }
        } else if (p->d_stlist) {   // stencil list (values streamed) and the other chunks (disjoint rows)
            // the small, latency-bound genlist walk runs beside the list kernel
            // on the plan's second stream when it has one (kSlistConcurrent)
            cudaStream_t gs = p->gside ? p->gside : st;
            if (p->gside && (cudaEventRecord(p->ev_gfork, st) != cudaSuccess ||
                             cudaStreamWaitEvent(p->gside, p->ev_gfork, 0) != cudaSuccess))
                return PEPP_E_CUDA;
            if (p->slist_long)
                pepp::k::sell_slist_kernel<kBlock, pepp::k::sell_slist_u<T, 16>(), 16, T><<<p->grid_slist, kBlock, 0, st>>>(
                    p->d_stlist, p->nstc, p->stab, (const T*)p->d_sval, x, y);
            else
                pepp::k::sell_slist_kernel<kBlock, pepp::k::sell_slist_u<T>(), 8, T><<<p->grid_slist, kBlock, 0, st>>>(
                    p->d_stlist, p->nstc, p->stab, (const T*)p->d_sval, x, y);
            if (p->ngen > 0)   // the genlist walk of the PAT instance, with no pattern chunks (phase A empty)
                pepp::k::sell_kernel<kBlock, false, true, T><<<p->grid_sell, kBlock, 0, gs>>>(
                    (int)p->nrows, p->ngen, p->d_chunk_ptr, p->d_chunk_len, p->d_rowlen, nullptr,
                    p->d_scol, p->d_scol16, p->d_soff, sell_pattern_table<T>(p), (const T*)p->d_sval, x, y, 1, nullptr,
                    nullptr, 0, p->d_genlist);
            if (p->gside && (cudaEventRecord(p->ev_gjoin, p->gside) != cudaSuccess ||
                             cudaStreamWaitEvent(st, p->ev_gjoin, 0) != cudaSuccess))
                return PEPP_E_CUDA;
        } else
            pepp::k::sell_kernel<kBlock, false, false, T><<<p->grid_sell, kBlock, 0, st>>>(
                (int)p->nrows, p->nchunks, p->d_chunk_ptr, p->d_chunk_len, p->d_rowlen, nullptr,
                p->d_scol, p->d_scol16, p->d_soff, pepp::k::NoPatterns{}, (const T*)p->d_sval, x, y, 1, nullptr,
                nullptr, 0, nullptr);
        if (p->nsell_mid)   // hybrid: the mid-length rows, after sell_kernel wrote 0 for them
            pepp::k::sell_mid_kernel<256, T><<<(p->nsell_mid + 7) / 8, 256, 0, st>>>(
                p->nsell_mid, p->d_sell_mid, p->d_rp, p->d_col, val, x, y);
        if (p->nsell_seg)   // hybrid: the long rows, after sell_kernel wrote 0 for them
            pepp::k::sell_long_kernel<256, T><<<p->nsell_seg, 256, 0, st>>>(
                p->d_sell_seg, p->d_sell_lrow, p->d_sell_cnt, (T*)p->d_sell_part, p->d_col, val, x, y);
        break;
    case PEPP_V_PANEL: {
        const PanelLayout* L = nullptr;
        for (const auto& pl : p->panels) if (pl.lg == c.param) L = &pl;
        if (!L) return PEPP_E_INVALID;
        if (cudaMemsetAsync(y, 0, sizeof(T) * p->nrows, st) != cudaSuccess) return PEPP_E_CUDA;
        for (int k = 0; k < L->npanels; ++k) {
            const int j0 = L->poff[k], j1 = L->poff[k + 1];
            if (j1 <= j0) continue;
            const int g = (int)std::min<int64_t>(((int64_t)j1 - j0 + 255) / 256, (int64_t)p->sm_count * 16);
            pepp::k::panel_kernel<T><<<g, 256, 0, st>>>(j0, j1, L->d_prow, L->d_pstart, L->d_pcol, (const T*)L->d_pval, x, y);
        }
        break;
    }
    default:
        return PEPP_E_INVALID;
    }
    return cudaGetLastError() == cudaSuccess ? PEPP_OK : PEPP_E_CUDA;
}

// kernels launch_t enqueues for candidate c (mirrors its conditions; the
// tile kernels run only on 16-byte aligned x and y)
int launches_for(const pepp_spmv_plan_t* p, const Candidate& c, const void* x, const void* y) {
    const bool al = ((((uintptr_t)x) | ((uintptr_t)y)) & 15) == 0;
    if (p->nrows == 0) return 0;
    switch (c.variant) {
    case PEPP_V_CSR_VECTOR: return 1;
    case PEPP_V_MERGE_PATH:
        if (c.param == kMergeWarpParam) return p->ntiles_w > 0 ? 2 + (p->nlongruns_w > 0) : 0;
        return p->ntiles > 0 ? 2 + (p->nlongruns > 0) : 0;
    case PEPP_V_CSR_STREAM: return p->nitems > 0 ? 1 + (p->nlong > 0) : 0;
    case PEPP_V_SELL:
        return (p->d_stlist ? (p->stl.ntiles && al ? 1 + (p->nstrest > 0) +
                                                         ((tile_walkers<true>() == 0 || !walkers_suffice<true>(p, p->stl)) && p->ngen > 0)
                                                   : 1 + (p->ngen > 0))
                            : (p->d_patlist && p->ptl.ntiles && al)
                                  ? 1 + ((tile_walkers<false>() == 0 || p->npatrest > 0 || !walkers_suffice<false>(p, p->ptl)) &&
                                         p->ngen + p->npatrest > 0)
                                  : 1) +
               (p->nsell_mid > 0) + (p->nsell_seg > 0);
    case PEPP_V_PANEL:
        for (const auto& pl : p->panels)
            if (pl.lg == c.param) {
                int k = 0;
                for (int i = 0; i < pl.npanels; ++i) k += pl.poff[i + 1] > pl.poff[i];
                return k;
            }
        return 0;
    default: return 0;
    }
}

// gather / scatter kernels one halo exchange launches (pack_unpack)
int halo_kernels(const pepp_spmv_plan_t* p) {
    int n = 0;
    for (const auto* v : {&p->send_x, &p->recv_x})
        for (const auto& t : *v) n += t.contig_start < 0 && t.count > 0;
    return n;
}

pepp_status_t launch(pepp_spmv_plan_t* p, const Candidate& c, const void* x, void* y, cudaStream_t st) {
    if (p->vt == PEPP_VALUE_F32) return launch_t<float>(p, c, (const float*)x, (float*)y, st);
    return launch_t<double>(p, c, (const double*)x, (double*)y, st);
}

// ---------------------------------------------------------------- history
void harvest(pepp_spmv_plan_t* p, bool block) {
    while (p->ring_count > 0) {
        TimingRec& r = p->ring[p->ring_head];
        if (block) cudaEventSynchronize(r.stop);
        cudaError_t q = cudaEventQuery(r.stop);
        if (q == cudaErrorNotReady) { (void)cudaGetLastError(); break; }
        float ms = 0.f;
        if (q == cudaSuccess && cudaEventElapsedTime(&ms, r.start, r.stop) == cudaSuccess) {
            // a candidate's first timed call in this plan is a warm-up, not a
            // sample: it can carry one-off costs (lazy module load of its
            // kernels, the SM clock ramping up from idle, cold TLBs) that, in
            // a 3-sample mean, once pushed the best candidate past a 1.7x
            // slower one on config 4 (round-2 bench, sell[1] vs csr_vector[2])
            if (r.cand >= 0 && r.cand < (int)p->warmed.size() && !p->warmed[r.cand]) p->warmed[r.cand] = 1;
            else pepp::history_add(p->hist, p->key, p->uids[r.cand], (double)ms * 1000.0);
        }
        (void)cudaGetLastError();
        r.pending = false;
        if (r.cand >= 0 && r.cand < (int)p->pending.size()) --p->pending[r.cand];
        p->ring_head = (p->ring_head + 1) % kTimingRing;
        --p->ring_count;
    }
}

int heuristic_candidate(const pepp_spmv_plan_t* p) {
    // use_history = 0: the argmin of the user's prediction function when it
    // predicted anything (ties -> lower index), else a fixed rule from the
    // context instance (mean, CV)
    {
        int c = -1;
        double best = 0.0;
        for (size_t i = 0; i < p->predicted.size(); ++i)
            if (p->eligible[i] && p->predicted[i] > 0 && (c < 0 || p->predicted[i] < best)) { c = (int)i; best = p->predicted[i]; }
        if (c >= 0) return c;
    }
    const double mean = p->info.mean_row, cv = p->info.cv_row;
    auto find = [&](int v, int prm) {
        for (size_t i = 0; i < p->cands.size(); ++i)
            if (p->cands[i].variant == v && (prm < 0 || p->cands[i].param == prm) && p->eligible[i]) return (int)i;
        return -1;
    };
    int c = -1;
    if (cv > 1.0) c = find(PEPP_V_MERGE_PATH, -1);
    if (c < 0 && mean <= 12.0 && cv <= 0.5) c = find(PEPP_V_SELL, -1);
    if (c < 0) {
        const int tpr = mean <= 6 ? 2 : mean <= 12 ? 4 : mean <= 24 ? 8 : mean <= 96 ? 16 : 32;
        c = find(PEPP_V_CSR_VECTOR, tpr);
    }
    for (size_t i = 0; c < 0 && i < p->cands.size(); ++i) if (p->eligible[i]) c = (int)i;
    return c;
}

void fill_choice(const pepp_spmv_plan_t* p, int cand, int calibrating, double pred, pepp_choice_t* out) {
    out->variant = p->cands[cand].variant;
    out->param = p->cands[cand].param;
    out->nparts = p->opts.nranks;
    out->exchange = p->exchange;
    out->calibrating = calibrating;
    out->candidate = cand;
    out->predicted_us = pred;
    out->layout_bytes = p->cand_bytes[cand];
}

// frozen: the call is being captured into a CUDA graph — no event queries (a
// global-mode capture forbids them) and no calibration (nothing is timed):
// the best measured candidate so far, else the heuristic
pepp_status_t select_choice(pepp_spmv_plan_t* p, pepp_choice_t* out, bool frozen = false) {
    if (!frozen) harvest(p, false);
    int calibrating = 0;
    double pred = 0.0;
    int cand;
    if (frozen) {
        cand = -1;
        for (int32_t c = 0; c < (int32_t)p->cands.size(); ++c) {
            const pepp::Welford* w = pepp::history_get(p->hist, p->key, p->uids[c]);
            if (!p->eligible[c] || !w || w->count == 0) continue;
            if (cand < 0 || w->mean < pred * 0.99) { cand = c; pred = w->mean; }
        }
        if (cand < 0) cand = heuristic_candidate(p);
    } else if (p->opts.use_history) {
        // Calibration counts timed calls already in flight, so the host (which
        // runs far ahead of the GPU) moves on to the next under-sampled
        // candidate instead of re-issuing the same one; once every candidate
        // has min_samples calls issued, wait for them once and exploit.
        const int32_t ms = std::max(1, p->opts.min_samples);
        const int32_t n = (int32_t)p->cands.size();
        auto hget = [&](int32_t c) { return pepp::history_get(p->hist, p->key, p->uids[c]); };
        double best_mean = -1.0, prior_best = -1.0;
        for (int32_t c = 0; c < n && !p->calibrated; ++c) {
            const pepp::Welford* w = hget(c);
            if (p->eligible[c] && w && w->count > 0 && (best_mean < 0 || w->mean < best_mean)) best_mean = w->mean;
            if (p->eligible[c] && p->prior[c] > 0 && (prior_best < 0 || p->prior[c] < prior_best)) prior_best = p->prior[c];
        }
        // ruled out: own samples > 4x the best own mean, or (never sampled) a
        // prior > 4x the best prior from the nearest recorded context
        auto ruled_out = [&](int32_t c, const pepp::Welford* w) {
            if (pepp::history_abandoned(w, best_mean)) return true;
            return (!w || w->count == 0) && prior_best > 0 && p->prior[c] > pepp::kAbandonFactor * prior_best;
        };
        auto rounds = [&]() {   // refinement only while two or more contenders exist
            int32_t k = 0;
            for (int32_t c = 0; c < n; ++c) k += p->eligible[c] && pepp::history_contender(hget(c), best_mean);
            return k >= 2 ? pepp::kRefineRounds * ms : ms;
        };
        cand = -1;
        // once calibration has finished it stays finished (sample counts only
        // grow): the per-call path skips the round scan (select < 1 µs)
        for (int32_t r = 1; !p->calibrated && r <= rounds() && cand < 0; ++r) {
            // round r: every candidate not yet ruled out gets its r-th timed call
            // (calls still in flight count, so the host can run ahead of the GPU);
            // rounds past ms refine only the contenders (within kContendFactor
            // of the best mean), as pepp::history_pick does
            for (int pass = 0; pass < 2 && cand < 0; ++pass) {
                bool waiting = false;
                for (int32_t oi = 0; oi < n; ++oi) {
                    const int32_t c = p->order[oi];
                    if (!p->eligible[c]) continue;
                    const pepp::Welford* w = hget(c);
                    if (ruled_out(c, w)) continue;
                    if (r > ms && !pepp::history_contender(w, best_mean)) continue;
                    const int64_t done = w ? w->count : 0;
                    if (done + p->pending[c] < r) {
                        cand = c; calibrating = 1;
                        pred = w && w->count ? w->mean : (p->prior[c] > 0 ? p->prior[c] : 0.0);
                        break;
                    }
                    if (done < r) waiting = true;
                }
                // the round is fully issued but not measured: wait for it once, so
                // the next round can rule out candidates from their timings
                if (cand < 0 && waiting) {
                    harvest(p, true);
                    best_mean = -1.0;
                    for (int32_t c = 0; c < n; ++c) {
                        const pepp::Welford* w = hget(c);
                        if (p->eligible[c] && w && w->count > 0 && (best_mean < 0 || w->mean < best_mean)) best_mean = w->mean;
                    }
                } else {
                    break;
                }
            }
        }
        if (cand < 0) {
            p->calibrated = true;
            // exploitation: argmin of the measured means, ties within 1 % -> lower index (A10)
            double bt = 0.0;
            for (int32_t c = 0; c < n; ++c) {
                const pepp::Welford* w = hget(c);
                if (!p->eligible[c] || !w || w->count == 0) continue;
                if (cand < 0 || w->mean < bt * 0.99) { cand = c; bt = w->mean; }
            }
            calibrating = 0;
            pred = bt;
        }
    } else {
        cand = heuristic_candidate(p);
    }
    if (cand < 0) return PEPP_E_INVALID;
    fill_choice(p, cand, calibrating, pred, out);
    return PEPP_OK;
}

// ---------------------------------------------------------------- NCCL
pepp_status_t nccl_ok(const pepp_spmv_plan_t* p, int r) { (void)p; return r == 0 ? PEPP_OK : PEPP_E_NCCL; }

int nccl_value_type(const pepp_spmv_plan_t* p) { return p->vt == PEPP_VALUE_F32 ? pepp::NCCL_FLOAT32 : pepp::NCCL_FLOAT64; }

// grouped broadcasts: block j = y[bounds[j], bounds[j+1]) from rank j to
// every rank of the plan's communicator (allgatherv of nb blocks, nb <= ranks)
pepp_status_t exchange_blocks(pepp_spmv_plan_t* p, const int64_t* bounds, int nb, void* y, cudaStream_t st) {
    PEPP_NVTX("pepp exchange allgatherv");
    const Nccl* n = p->nccl;
    char* yb = (char*)y;
    if (nccl_ok(p, n->GroupStart())) return PEPP_E_NCCL;
    for (int r = 0; r < nb; ++r) {
        const int64_t b = bounds[r], cnt = bounds[r + 1] - b;
        if (cnt == 0) continue;
        char* at = yb + b * (int64_t)p->esz;
        if (n->Broadcast(at, at, (size_t)cnt, nccl_value_type(p), r, p->comm, st)) { n->GroupEnd(); return PEPP_E_NCCL; }
    }
    return nccl_ok(p, n->GroupEnd());
}

pepp_status_t exchange_allgather(pepp_spmv_plan_t* p, void* y, cudaStream_t st) {
    return exchange_blocks(p, p->row_bounds.data(), p->opts.nranks, y, st);
}

template <typename T>
void pack_unpack(std::vector<PeerXfer>& lst, T* y, bool pack, cudaStream_t st) {
    for (auto& t : lst) {
        if (t.contig_start >= 0 || t.count == 0) continue;
        const int g = (int)std::min<int64_t>(1024, (t.count + 255) / 256);
        if (pack) pepp::k::gather_kernel<T><<<g, 256, 0, st>>>(t.count, t.d_idx, y, (T*)t.d_buf);
        else pepp::k::scatter_kernel<T><<<g, 256, 0, st>>>(t.count, t.d_idx, (const T*)t.d_buf, y);
    }
}

// point-to-point transfer lists (halo ghosts, or a distribution's scatter):
// pack scattered send entries, grouped send/recv, unpack scattered receives
pepp_status_t exchange_xfer(pepp_spmv_plan_t* p, std::vector<PeerXfer>& recv, std::vector<PeerXfer>& send, void* y,
                            cudaStream_t st) {
    const Nccl* n = p->nccl;
    char* yb = (char*)y;
    const int64_t es = (int64_t)p->esz;
    if (p->vt == PEPP_VALUE_F32) pack_unpack<float>(send, (float*)y, true, st);
    else pack_unpack<double>(send, (double*)y, true, st);
    if (n->GroupStart()) return PEPP_E_NCCL;
    for (auto& t : send) {
        if (!t.count) continue;
        const void* src = t.contig_start >= 0 ? (const void*)(yb + t.contig_start * es) : t.d_buf;
        if (n->Send(src, (size_t)t.count, nccl_value_type(p), t.peer, p->comm, st)) { n->GroupEnd(); return PEPP_E_NCCL; }
    }
    for (auto& t : recv) {
        if (!t.count) continue;
        void* dst = t.contig_start >= 0 ? (void*)(yb + t.contig_start * es) : t.d_buf;
        if (n->Recv(dst, (size_t)t.count, nccl_value_type(p), t.peer, p->comm, st)) { n->GroupEnd(); return PEPP_E_NCCL; }
    }
    if (n->GroupEnd()) return PEPP_E_NCCL;
    if (p->vt == PEPP_VALUE_F32) pack_unpack<float>(recv, (float*)y, false, st);
    else pack_unpack<double>(recv, (double*)y, false, st);
    return cudaGetLastError() == cudaSuccess ? PEPP_OK : PEPP_E_CUDA;
}

pepp_status_t exchange_halo(pepp_spmv_plan_t* p, void* y, cudaStream_t st) {
    PEPP_NVTX("pepp exchange halo");
    return exchange_xfer(p, p->recv_x, p->send_x, y, st);
}

// plan-time halo setup: ghosts (what I receive) from my columns; what I send
// is learnt from the peers with one NCCL exchange of counts and indices.
pepp_status_t setup_halo(pepp_spmv_plan_t* p, const std::vector<int32_t>& ghosts, cudaStream_t st) {
    const int P = p->opts.nranks, me = p->opts.rank;
    std::vector<int64_t> rcount(P, 0), scount(P, 0);
    std::vector<std::vector<int32_t>> rlist(P);
    for (int32_t c : ghosts) {
        int q = (int)(std::upper_bound(p->row_bounds.begin(), p->row_bounds.end(), (int64_t)c) - p->row_bounds.begin()) - 1;
        rlist[q].push_back(c);
    }
    for (int q = 0; q < P; ++q) rcount[q] = (int64_t)rlist[q].size();
    // exchange counts: send rcount[q] to q, receive scount[q] from q
    DevTmp<int64_t> d_rc, d_sc;
    PEPP_CUDA_TRY(d_rc.alloc(P));
    PEPP_CUDA_TRY(d_sc.alloc(P));
    PEPP_CUDA_TRY(cudaMemcpy(d_rc.p, rcount.data(), sizeof(int64_t) * P, cudaMemcpyHostToDevice));
    PEPP_CUDA_TRY(cudaMemset(d_sc.p, 0, sizeof(int64_t) * P));
    const Nccl* n = p->nccl;
    if (n->GroupStart()) return PEPP_E_NCCL;
    for (int q = 0; q < P; ++q) {
        if (q == me) continue;
        n->Send(d_rc.p + q, 1, pepp::NCCL_INT64, q, p->comm, st);
        n->Recv(d_sc.p + q, 1, pepp::NCCL_INT64, q, p->comm, st);
    }
    if (n->GroupEnd()) return PEPP_E_NCCL;
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    PEPP_CUDA_TRY(cudaMemcpy(scount.data(), d_sc.p, sizeof(int64_t) * P, cudaMemcpyDeviceToHost));
    scount[me] = 0;
    // exchange index lists
    std::vector<DevTmp<int>> d_r(P), d_s(P);
    for (int q = 0; q < P; ++q) {
        if (rcount[q]) {
            PEPP_CUDA_TRY(d_r[q].alloc(rcount[q]));
            PEPP_CUDA_TRY(cudaMemcpy(d_r[q].p, rlist[q].data(), sizeof(int) * rcount[q], cudaMemcpyHostToDevice));
        }
        if (scount[q]) PEPP_CUDA_TRY(d_s[q].alloc(scount[q]));
    }
    if (n->GroupStart()) return PEPP_E_NCCL;
    for (int q = 0; q < P; ++q) {
        if (rcount[q]) n->Send(d_r[q].p, (size_t)rcount[q], pepp::NCCL_INT32, q, p->comm, st);
        if (scount[q]) n->Recv(d_s[q].p, (size_t)scount[q], pepp::NCCL_INT32, q, p->comm, st);
    }
    if (n->GroupEnd()) return PEPP_E_NCCL;
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    auto make = [&](int q, std::vector<int32_t>& lst, DevTmp<int>& d_list, std::vector<PeerXfer>& out) -> pepp_status_t {
        PeerXfer t;
        t.peer = q;
        t.count = (int64_t)lst.size();
        const bool contig = !lst.empty() && (int64_t)lst.back() - lst.front() + 1 == t.count;
        t.contig_start = contig ? lst.front() : -1;
        if (!contig && t.count) {
            DevTmp<double> buf;   // 8-byte slots hold either value type
            PEPP_CUDA_TRY(buf.alloc(t.count));
            t.d_idx = d_list.release();
            t.d_buf = buf.release();
        }
        out.push_back(t);
        return PEPP_OK;
    };
    for (int q = 0; q < P; ++q) {
        if (rcount[q]) { pepp_status_t s = make(q, rlist[q], d_r[q], p->recv_x); if (s) return s; }
        if (scount[q]) {
            std::vector<int32_t> sl(scount[q]);
            PEPP_CUDA_TRY(cudaMemcpy(sl.data(), d_s[q].p, sizeof(int) * scount[q], cudaMemcpyDeviceToHost));
            int64_t lo = INT64_MAX, hi = INT64_MIN;
            for (int32_t v : sl) {
                p->send_local.push_back((int64_t)v - p->row_offset);
                lo = std::min<int64_t>(lo, (int64_t)v - p->row_offset);
                hi = std::max<int64_t>(hi, (int64_t)v - p->row_offset + 1);
            }
            p->send_rng.push_back({q, lo, hi});
            pepp_status_t s = make(q, sl, d_s[q], p->send_x);
            if (s) return s;
        }
    }
    int64_t tr = 0, ts = 0;
    for (auto& t : p->recv_x) tr += t.count;
    for (auto& t : p->send_x) ts += t.count;
    p->info.halo_recv = tr;
    p->info.halo_send = ts;
    return PEPP_OK;
}

// Transfer lists for `needed` (sorted distinct global rows this rank must
// hold after a call) whose owners are the blocks [bounds[q], bounds[q+1]),
// q < nb: one count and one index exchange over the plan's communicator
// (every rank takes part, also ranks that need nothing), as in setup_halo.
pepp_status_t setup_xfer(pepp_spmv_plan_t* p, const std::vector<int32_t>& needed, const std::vector<int64_t>& bounds,
                         std::vector<PeerXfer>& recv, std::vector<PeerXfer>& send, cudaStream_t st) {
    const int P = p->opts.nranks, me = p->opts.rank;
    std::vector<int64_t> rcount(P, 0), scount(P, 0);
    std::vector<std::vector<int32_t>> rlist(P);
    for (int32_t c : needed) {
        const int q = (int)(std::upper_bound(bounds.begin(), bounds.end(), (int64_t)c) - bounds.begin()) - 1;
        if (q >= 0 && q < P && q != me) rlist[q].push_back(c);
    }
    for (int q = 0; q < P; ++q) rcount[q] = (int64_t)rlist[q].size();
    DevTmp<int64_t> d_rc, d_sc;
    PEPP_CUDA_TRY(d_rc.alloc(P));
    PEPP_CUDA_TRY(d_sc.alloc(P));
    PEPP_CUDA_TRY(cudaMemcpy(d_rc.p, rcount.data(), sizeof(int64_t) * P, cudaMemcpyHostToDevice));
    PEPP_CUDA_TRY(cudaMemset(d_sc.p, 0, sizeof(int64_t) * P));
    const Nccl* n = p->nccl;
    if (n->GroupStart()) return PEPP_E_NCCL;
    for (int q = 0; q < P; ++q) {
        if (q == me) continue;
        n->Send(d_rc.p + q, 1, pepp::NCCL_INT64, q, p->comm, st);
        n->Recv(d_sc.p + q, 1, pepp::NCCL_INT64, q, p->comm, st);
    }
    if (n->GroupEnd()) return PEPP_E_NCCL;
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    PEPP_CUDA_TRY(cudaMemcpy(scount.data(), d_sc.p, sizeof(int64_t) * P, cudaMemcpyDeviceToHost));
    scount[me] = 0;
    std::vector<DevTmp<int>> d_r(P), d_s(P);
    for (int q = 0; q < P; ++q) {
        if (rcount[q]) {
            PEPP_CUDA_TRY(d_r[q].alloc(rcount[q]));
            PEPP_CUDA_TRY(cudaMemcpy(d_r[q].p, rlist[q].data(), sizeof(int) * rcount[q], cudaMemcpyHostToDevice));
        }
        if (scount[q]) PEPP_CUDA_TRY(d_s[q].alloc(scount[q]));
    }
    if (n->GroupStart()) return PEPP_E_NCCL;
    for (int q = 0; q < P; ++q) {
        if (rcount[q]) n->Send(d_r[q].p, (size_t)rcount[q], pepp::NCCL_INT32, q, p->comm, st);
        if (scount[q]) n->Recv(d_s[q].p, (size_t)scount[q], pepp::NCCL_INT32, q, p->comm, st);
    }
    if (n->GroupEnd()) return PEPP_E_NCCL;
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    auto make = [&](int q, const std::vector<int32_t>& lst, DevTmp<int>& d_list, std::vector<PeerXfer>& out) -> pepp_status_t {
        PeerXfer t;
        t.peer = q;
        t.count = (int64_t)lst.size();
        const bool contig = !lst.empty() && (int64_t)lst.back() - lst.front() + 1 == t.count;
        t.contig_start = contig ? lst.front() : -1;
        if (!contig && t.count) {
            DevTmp<double> buf;   // 8-byte slots hold either value type
            PEPP_CUDA_TRY(buf.alloc(t.count));
            t.d_idx = d_list.release();
            t.d_buf = buf.release();
        }
        out.push_back(t);
        return PEPP_OK;
    };
    for (int q = 0; q < P; ++q) {
        if (rcount[q]) { pepp_status_t s = make(q, rlist[q], d_r[q], recv); if (s) return s; }
        if (scount[q]) {
            std::vector<int32_t> sl(scount[q]);
            PEPP_CUDA_TRY(cudaMemcpy(sl.data(), d_s[q].p, sizeof(int) * scount[q], cudaMemcpyDeviceToHost));
            pepp_status_t s = make(q, sl, d_s[q], send);
            if (s) return s;
        }
    }
    return PEPP_OK;
}

int xfer_kernels(const std::vector<PeerXfer>& recv, const std::vector<PeerXfer>& send) {
    int n = 0;
    for (const auto* v : {&send, &recv})
        for (const auto& t : *v) n += t.contig_start < 0 && t.count > 0;
    return n;
}

pepp_status_t plan_impl(const pepp_csr_t* A, const pepp_spmv_opts_t* o, pepp_spmv_plan_t* p);

// rows [r0, r1) of this block as a plan of their own (unpartitioned, same
// options); the slice shares A's arrays, offset by row_ptr[r0] - first
pepp_status_t make_sub(const pepp_csr_t* A, const pepp_spmv_opts_t* o, const pepp_spmv_plan_t* p, int64_t r0,
                       int64_t r1, int reserve, pepp_spmv_plan_t** out) {
    *out = nullptr;
    int64_t b0 = 0, b1 = 0;
    if (A->on_device) {
        PEPP_CUDA_TRY(cudaMemcpy(&b0, A->row_ptr + r0, sizeof(int64_t), cudaMemcpyDeviceToHost));
        PEPP_CUDA_TRY(cudaMemcpy(&b1, A->row_ptr + r1, sizeof(int64_t), cudaMemcpyDeviceToHost));
    } else {
        b0 = A->row_ptr[r0];
        b1 = A->row_ptr[r1];
    }
    pepp_csr_t S = *A;
    S.nrows = r1 - r0;
    S.nnz = b1 - b0;
    S.first = b0;
    S.row_ptr = A->row_ptr + r0;
    if (A->nnz) {
        S.col_idx = A->col_idx + (b0 - A->first);
        S.values = (const char*)A->values + (b0 - A->first) * (int64_t)p->esz;
    }
    pepp_spmv_opts_t so = *o;
    so.nranks = 1; so.rank = 0; so.row_bounds = nullptr;
    so.nccl_comm = nullptr; so.nccl_unique_id = nullptr; so.exchange = PEPP_X_NONE;
    so.history_path = nullptr; so.overlap = 0;
    so.validate = 0;          // the whole block was validated
    so.device = p->device;
    pepp_spmv_plan_t* q = new (std::nothrow) pepp_spmv_plan_t();
    if (!q) return PEPP_E_NOMEM;
    q->device = -1;
    q->reserve_sms = reserve;
    pepp_status_t s = plan_impl(&S, &so, q);
    if (s) { free_plan(q); return s; }
    *out = q;
    return PEPP_OK;
}

// Overlap of the halo exchange with the interior rows (opts.overlap). The
// rows peers receive must lie in a head [0, h) and a tail [R - t, R) with
// h + t <= R / 2; else the block keeps the in-order kernel -> exchange path.
pepp_status_t setup_overlap(const pepp_csr_t* A, const pepp_spmv_opts_t* o, pepp_spmv_plan_t* p) {
    const int64_t R = p->nrows;
    int64_t h = 0, t = 0;
    for (int64_t v : p->send_local) {
        if (v < 0 || v >= R) return PEPP_OK;   // not a row of this block: no overlap
        if (v < R / 2) h = std::max(h, v + 1);
        else t = std::max(t, R - v);
    }
    if (R < 2 || h + t > R / 2) return PEPP_OK;
    pepp_status_t s;
    const int64_t bnd[4] = {0, h, R - t, R};
    for (int i = 0; i < 3; ++i) {
        p->sub_r0[i] = bnd[i];
        if (bnd[i + 1] > bnd[i] && (s = make_sub(A, o, p, bnd[i], bnd[i + 1], i == 1 ? kReserveSms : 0, &p->sub[i])))
            return s;
    }
    int lo = 0, hi = 0;
    PEPP_CUDA_TRY(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    PEPP_CUDA_TRY(cudaStreamCreateWithPriority(&p->side, cudaStreamNonBlocking, hi));
    PEPP_CUDA_TRY(cudaEventCreateWithFlags(&p->ev_fork, cudaEventDisableTiming));
    PEPP_CUDA_TRY(cudaEventCreateWithFlags(&p->ev_join, cudaEventDisableTiming));
    p->info.overlap = 1;
    p->info.overlap_head = h;
    p->info.overlap_tail = t;
    return PEPP_OK;
}

// ---------------------------------------------------------------- P2P
// Fused peer-memory halo (pepp_spmv_p2p_buffers): symmetric buffers and a
// signal block per rank, exported with CUDA IPC, their handles all-gathered
// over the plan's communicator (grouped broadcasts of bytes), the peers' ones
// opened (cudaIpcMemLazyEnablePeerAccess: NVLink / NVSwitch mappings).
struct P2PHandles {
    cudaIpcMemHandle_t buf[kP2PMaxBuf];
    cudaIpcMemHandle_t sig;
    int64_t ok;                              // 1 = this rank's export succeeded
};

// max over ranks of v (an all-reduce that doubles as a barrier)
pepp_status_t nccl_allmax(pepp_spmv_plan_t* p, cudaStream_t st, int64_t* v) {
    DevTmp<int64_t> d;
    PEPP_CUDA_TRY(d.alloc(1));
    PEPP_CUDA_TRY(cudaMemcpyAsync(d.p, v, sizeof(int64_t), cudaMemcpyHostToDevice, st));
    if (p->nccl->AllReduce(d.p, d.p, 1, pepp::NCCL_INT64, pepp::NCCL_OP_MAX, p->comm, st)) return PEPP_E_NCCL;
    PEPP_CUDA_TRY(cudaMemcpyAsync(v, d.p, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    return PEPP_OK;
}

pepp_status_t nccl_barrier(pepp_spmv_plan_t* p, cudaStream_t st) {
    int64_t v = 0;
    return nccl_allmax(p, st, &v);
}

// elementwise max over ranks of a host vector of doubles (agreement on times)
pepp_status_t nccl_allmax_f64(pepp_spmv_plan_t* p, cudaStream_t st, std::vector<double>& v) {
    if (v.empty()) return PEPP_OK;
    DevTmp<double> d;
    PEPP_CUDA_TRY(d.alloc(v.size()));
    PEPP_CUDA_TRY(cudaMemcpyAsync(d.p, v.data(), sizeof(double) * v.size(), cudaMemcpyHostToDevice, st));
    if (p->nccl->AllReduce(d.p, d.p, v.size(), pepp::NCCL_FLOAT64, pepp::NCCL_OP_MAX, p->comm, st)) return PEPP_E_NCCL;
    PEPP_CUDA_TRY(cudaMemcpyAsync(v.data(), d.p, sizeof(double) * v.size(), cudaMemcpyDeviceToHost, st));
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    return PEPP_OK;
}

// every rank's value of v (grouped broadcasts of one int64 per rank)
pepp_status_t nccl_allgather_i64(pepp_spmv_plan_t* p, cudaStream_t st, int64_t v, std::vector<int64_t>& all) {
    const int P = p->opts.nranks, me = p->opts.rank;
    all.assign(P, 0);
    all[me] = v;
    DevTmp<int64_t> d;
    PEPP_CUDA_TRY(d.alloc(P));
    PEPP_CUDA_TRY(cudaMemcpyAsync(d.p, all.data(), sizeof(int64_t) * P, cudaMemcpyHostToDevice, st));
    if (p->nccl->GroupStart()) return PEPP_E_NCCL;
    for (int r = 0; r < P; ++r)
        if (p->nccl->Broadcast(d.p + r, d.p + r, 1, pepp::NCCL_INT64, r, p->comm, st)) { p->nccl->GroupEnd(); return PEPP_E_NCCL; }
    if (p->nccl->GroupEnd()) return PEPP_E_NCCL;
    PEPP_CUDA_TRY(cudaMemcpyAsync(all.data(), d.p, sizeof(int64_t) * P, cudaMemcpyDeviceToHost, st));
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    return PEPP_OK;
}

pepp_status_t plan_impl(const pepp_csr_t* A, const pepp_spmv_opts_t* o, pepp_spmv_plan_t* p);

// Distribution candidates P' < nranks (opts.dist_select; §8(a) a4 "P" and
// §V-D P@38827 "which ... device to use ... data locality and potential
// data-transfer cost"). For every P' = 2^i dividing nranks (and whose blocks
// fit the int32 device indexing), P'-block j is the union of the nranks/P'
// consecutive row blocks j*k .. j*k+k-1 (k = nranks/P'; its boundaries are
// row_bounds[j*k], so with the A9 rule they are exactly A9's P'-way split).
// Each rank ships its block (narrowed row pointer, columns, values) to rank
// r / k over NCCL; rank j < P' widens the row pointers to one union row
// pointer and plans the union (P' ranks, halo exchange among them). Every
// rank then learns, for the HALO form, where its own rows and own ghosts
// come from after a P' call (setup_xfer). Collective over all ranks.
pepp_status_t setup_dist_parts(const pepp_spmv_opts_t* o, pepp_spmv_plan_t* p, const std::vector<int32_t>& ghosts,
                               cudaStream_t st) {
    const int N = o->nranks, me = o->rank;
    const int64_t es = (int64_t)p->esz;
    std::vector<int64_t> nnz_all, pad_all;
    pepp_status_t s;
    if ((s = nccl_allgather_i64(p, st, p->nnz, nnz_all))) return s;
    if ((s = nccl_allgather_i64(p, st, p->pad, pad_all))) return s;
    p->global_nnz = 0;
    for (int64_t z : nnz_all) p->global_nnz += z;
    for (int parts = 1; parts < N; parts *= 2) {
        if (N % parts) continue;
        const int k = N / parts;
        bool fits = true;   // the same verdict on every rank (global facts only)
        for (int j = 0; j < parts; ++j) {
            int64_t z = 0;
            for (int r = j * k; r < (j + 1) * k; ++r) z += nnz_all[r];
            fits &= z + 8 < (int64_t)INT32_MAX && p->row_bounds[(j + 1) * k] - p->row_bounds[j * k] < (int64_t)INT32_MAX;
        }
        if (!fits) continue;
        DistPart dp;
        dp.parts = parts;
        dp.bounds.resize(parts + 1);
        for (int j = 0; j <= parts; ++j) dp.bounds[j] = p->row_bounds[(int64_t)j * k];
        // ---- ship the blocks: rank r -> rank r / k
        const int dest = me / k;
        const bool recv_side = me < parts;
        int64_t urows = 0, unnz = 0;
        std::vector<int64_t> zoff(k + 1, 0);   // union nonzero offset of each source block
        if (recv_side) {
            urows = dp.bounds[me + 1] - dp.bounds[me];
            for (int i = 0; i < k; ++i) zoff[i + 1] = zoff[i] + nnz_all[me * k + i];
            unnz = zoff[k];
        }
        DevTmp<int64_t> u_rp;
        DevTmp<int> u_col;
        DevTmp<unsigned char> u_val;
        std::vector<DevTmp<int>> rp32(k);
        if (recv_side) {
            PEPP_CUDA_TRY(u_rp.alloc(urows + 1));
            PEPP_CUDA_TRY(u_col.alloc(unnz));
            PEPP_CUDA_TRY(u_val.alloc((size_t)std::max<int64_t>(1, unnz) * es));
            for (int i = 0; i < k; ++i) {
                const int src = me * k + i;
                PEPP_CUDA_TRY(rp32[i].alloc(p->row_bounds[src + 1] - p->row_bounds[src] + 1));
            }
        }
        const Nccl* n = p->nccl;
        if (n->GroupStart()) return PEPP_E_NCCL;
        if (dest != me) {
            n->Send(p->d_rp, (size_t)(p->nrows + 1), pepp::NCCL_INT32, dest, p->comm, st);
            if (p->nnz) {
                n->Send(p->d_col + p->pad, (size_t)p->nnz, pepp::NCCL_INT32, dest, p->comm, st);
                n->Send((char*)p->d_val + p->pad * es, (size_t)(p->nnz * es), pepp::NCCL_INT8, dest, p->comm, st);
            }
        }
        if (recv_side) {
            for (int i = 0; i < k; ++i) {
                const int src = me * k + i;
                const int64_t rows = p->row_bounds[src + 1] - p->row_bounds[src], z = nnz_all[src];
                if (src == me) {   // this rank's own block is part of its union (j = 0 only)
                    PEPP_CUDA_TRY(cudaMemcpyAsync(rp32[i].p, p->d_rp, sizeof(int) * (rows + 1), cudaMemcpyDeviceToDevice, st));
                    if (z) {
                        PEPP_CUDA_TRY(cudaMemcpyAsync(u_col.p + zoff[i], p->d_col + p->pad, sizeof(int) * z, cudaMemcpyDeviceToDevice, st));
                        PEPP_CUDA_TRY(cudaMemcpyAsync(u_val.p + zoff[i] * es, (char*)p->d_val + p->pad * es, (size_t)(z * es),
                                                      cudaMemcpyDeviceToDevice, st));
                    }
                    continue;
                }
                n->Recv(rp32[i].p, (size_t)(rows + 1), pepp::NCCL_INT32, src, p->comm, st);
                if (z) {
                    n->Recv(u_col.p + zoff[i], (size_t)z, pepp::NCCL_INT32, src, p->comm, st);
                    n->Recv(u_val.p + zoff[i] * es, (size_t)(z * es), pepp::NCCL_INT8, src, p->comm, st);
                }
            }
        }
        if (n->GroupEnd()) return PEPP_E_NCCL;
        PEPP_CUDA_TRY(cudaStreamSynchronize(st));
        if (recv_side) {
            // union row pointer: block i's rows at union row offset ro, entries
            // rebased from (local offset + pad_src) to zoff[i]; the last entry
            // of one block is the first of the next (same value), so the
            // blocks are written in order and each writes rows + 1 entries
            int64_t ro = 0;
            for (int i = 0; i < k; ++i) {
                const int src = me * k + i;
                const int64_t rows = p->row_bounds[src + 1] - p->row_bounds[src];
                const int g = (int)std::min<int64_t>(1024, (rows + 1 + 255) / 256);
                pepp::k::rowptr_widen_kernel<<<g, 256, 0, st>>>(rows + 1, rp32[i].p, zoff[i] - pad_all[src], u_rp.p + ro);
                PEPP_CUDA_TRY(cudaGetLastError());
                PEPP_CUDA_TRY(cudaStreamSynchronize(st));
                ro += rows;
            }
            pepp_csr_t U{};
            U.nrows = urows;
            U.ncols = p->ncols;
            U.nnz = unnz;
            U.first = 0;
            U.row_ptr = u_rp.p;
            U.col_idx = u_col.p;
            U.values = u_val.p;
            U.on_device = 1;
            U.value_type = p->vt;
            pepp_spmv_opts_t so = *o;
            so.nranks = parts;
            so.rank = me;
            so.row_bounds = parts > 1 ? dp.bounds.data() : nullptr;
            so.nccl_comm = parts > 1 ? (void*)p->comm : nullptr;
            so.nccl_unique_id = nullptr;
            so.exchange = parts > 1 ? PEPP_X_HALO : PEPP_X_NONE;   // explicit: no AUTO all-reduce among a subset
            so.history_path = nullptr;
            so.overlap = 0;
            so.validate = 0;
            so.dist_select = 0;
            so.device = p->device;
            pepp_spmv_plan_t* q = new (std::nothrow) pepp_spmv_plan_t();
            s = q ? PEPP_OK : PEPP_E_NOMEM;
            if (q) {
                q->device = -1;
                if ((s = plan_impl(&U, &so, q))) { free_plan(q); q = nullptr; }
            }
            dp.plan = q;
        }
        {   // agreement: a rank whose P' plan failed (e.g. out of memory for the union of
            // its blocks) must not leave the others inside the next collectives
            int64_t code = -(int64_t)s;
            const pepp_status_t sa = nccl_allmax(p, st, &code);
            if (sa || code) {
                free_plan(dp.plan);
                return sa ? sa : (s ? s : (pepp_status_t)(-code));
            }
        }
        p->dparts.push_back(std::move(dp));   // owned by the plan from here on (freed with it)
        // ---- HALO form: own rows + own ghosts from their P' owners
        {
            DistPart& D = p->dparts.back();
            std::vector<int32_t> need;
            const int64_t lo = p->row_offset, hi = p->row_offset + p->nrows;
            const int64_t clo = recv_side ? D.bounds[me] : 0, chi = recv_side ? D.bounds[me + 1] : 0;
            need.reserve(p->nrows + ghosts.size());
            size_t gi = 0;
            auto add = [&](int64_t r) { if (r < clo || r >= chi) need.push_back((int32_t)r); };
            for (int64_t r = lo; r < hi; ++r) {
                while (gi < ghosts.size() && ghosts[gi] < r) add(ghosts[gi++]);
                add(r);
            }
            while (gi < ghosts.size()) add(ghosts[gi++]);
            if ((s = setup_xfer(p, need, D.bounds, D.recv_x, D.send_x, st))) return s;
            // gather form: after a P' = nranks call (own rows + own ghosts
            // valid), what a P' call on this rank reads on top of that — the
            // rest of its P' block and its P' ghosts — from their owners
            std::vector<int32_t> gneed;
            if (recv_side && D.plan) {
                std::vector<int32_t> pcols(D.plan->nnz), pghost;
                if (D.plan->nnz)
                    PEPP_CUDA_TRY(cudaMemcpy(pcols.data(), D.plan->d_col + D.plan->pad, sizeof(int) * D.plan->nnz,
                                             cudaMemcpyDeviceToHost));
                pepp::halo_ghost_list(pcols.data(), D.plan->nnz, clo, chi, pghost);
                auto held = [&](int64_t r) {
                    return (r >= lo && r < hi) || std::binary_search(ghosts.begin(), ghosts.end(), (int32_t)r);
                };
                size_t pg = 0;
                for (int64_t r = clo; r < chi || pg < pghost.size();) {
                    int64_t nxt;
                    if (pg < pghost.size() && (r >= chi || pghost[pg] < r)) nxt = pghost[pg++];
                    else nxt = r++;
                    if (!held(nxt)) gneed.push_back((int32_t)nxt);
                }
                std::sort(gneed.begin(), gneed.end());
                gneed.erase(std::unique(gneed.begin(), gneed.end()), gneed.end());
            }
            if ((s = setup_xfer(p, gneed, p->row_bounds, D.recv_g, D.send_g, st))) return s;
        }
    }
    return PEPP_OK;
}

// after a NEXT_INPUT exchange that ran with P'' = `parts_done` partitions:
// when the plan's chosen distribution for NEXT_INPUT calls is a P' < nranks
// other than P'', bring what a P' call reads to the P' ranks (the gather
// lists), so that y serves the plan's next call whichever path it takes
pepp_status_t dist_complete(pepp_spmv_plan_t* p, void* y, cudaStream_t st, int parts_done, int* launches) {
    if (p->dist_next < 0) return PEPP_OK;
    const int parts = p->dcands[p->dist_next].parts;
    if (parts == p->opts.nranks || parts == parts_done) return PEPP_OK;
    for (auto& dp : p->dparts)
        if (dp.parts == parts) {
            if (launches) *launches += xfer_kernels(dp.recv_g, dp.send_g);
            return exchange_xfer(p, dp.recv_g, dp.send_g, y, st);
        }
    return PEPP_OK;
}

// undo a registration every rank agreed had failed: nothing of it is in use
// on any rank, so the plan stays usable with the NCCL halo
void p2p_reset(pepp_spmv_plan_t* p) {
    for (void* m : p->p2p_opened) cudaIpcCloseMemHandle(m);
    p->p2p_opened.clear();
    for (void*& b : p->p2p_buf)
        if (b) { cudaFree(b); b = nullptr; p->dev_bytes -= p->global_rows * (int64_t)p->esz; }
    if (p->d_sig) { cudaFree(p->d_sig); p->d_sig = nullptr; p->dev_bytes -= (int64_t)sizeof(unsigned long long) * (2 * p->opts.nranks + 2); }
    if (p->h_err) { cudaFreeHost(p->h_err); p->h_err = nullptr; }
    p->d_err = nullptr;
    p->p2p_nbuf = p->p2p_npush = p->p2p_nsend = p->p2p_nrecv = 0;
    (void)cudaGetLastError();
}

// this rank's half: buffers, signal block, error flag, IPC export
pepp_status_t p2p_export(pepp_spmv_plan_t* p, int nbuf, cudaStream_t st, P2PHandles* mine) {
    const int P = p->opts.nranks;
    pepp_status_t s;
    // test-only fault injection (tests/test_gpu_partitioned.py): this rank's
    // export fails, so every rank must return the error and fall back
    if (const char* f = std::getenv("PEPP_FAULT_P2P_EXPORT"))
        if (std::atoi(f) == p->opts.rank) { pepp::set_last_error("injected export failure", "PEPP_FAULT_P2P_EXPORT", __LINE__); return PEPP_E_CUDA; }
    if (!p->side) {   // a rank without a head / tail split (it sends nothing) still forks a side stream
        int lo = 0, hi = 0;
        PEPP_CUDA_TRY(cudaDeviceGetStreamPriorityRange(&lo, &hi));
        PEPP_CUDA_TRY(cudaStreamCreateWithPriority(&p->side, cudaStreamNonBlocking, hi));
        PEPP_CUDA_TRY(cudaEventCreateWithFlags(&p->ev_fork, cudaEventDisableTiming));
        PEPP_CUDA_TRY(cudaEventCreateWithFlags(&p->ev_join, cudaEventDisableTiming));
    }
    // symmetric buffers + signal block (zeroed before any peer can see them)
    for (int b = 0; b < nbuf; ++b) {
        if ((s = dalloc_bytes(p, &p->p2p_buf[b], p->global_rows * (int64_t)p->esz))) return s;
        PEPP_CUDA_TRY(cudaMemsetAsync(p->p2p_buf[b], 0, p->global_rows * p->esz, st));
    }
    if ((s = dalloc(p, &p->d_sig, 2 * (int64_t)P + 2))) return s;
    PEPP_CUDA_TRY(cudaMemsetAsync(p->d_sig, 0, sizeof(unsigned long long) * (2 * P + 2), st));
    PEPP_CUDA_TRY(cudaHostAlloc((void**)&p->h_err, sizeof(int), cudaHostAllocMapped));
    *p->h_err = 0;
    PEPP_CUDA_TRY(cudaHostGetDevicePointer((void**)&p->d_err, p->h_err, 0));
    for (int b = 0; b < nbuf; ++b) PEPP_CUDA_TRY(cudaIpcGetMemHandle(&mine->buf[b], p->p2p_buf[b]));
    PEPP_CUDA_TRY(cudaIpcGetMemHandle(&mine->sig, p->d_sig));
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    mine->ok = 1;
    return PEPP_OK;
}

// map the send-peers' buffers and the signal blocks of send and receive peers; build the push ranges
pepp_status_t p2p_import(pepp_spmv_plan_t* p, int nbuf, const std::vector<P2PHandles>& all) {
    const int P = p->opts.nranks, me = p->opts.rank;
    std::vector<int> sendp, recvp;   // peers this rank writes to (its send list) / receives from
    for (auto& t : p->send_x) if (t.count) sendp.push_back(t.peer);
    for (auto& t : p->recv_x) if (t.count) recvp.push_back(t.peer);
    std::sort(sendp.begin(), sendp.end());
    sendp.erase(std::unique(sendp.begin(), sendp.end()), sendp.end());
    std::sort(recvp.begin(), recvp.end());
    recvp.erase(std::unique(recvp.begin(), recvp.end()), recvp.end());
    if ((int)sendp.size() > pepp::k::kP2PMaxPeers || (int)recvp.size() > pepp::k::kP2PMaxPeers) return PEPP_E_UNSUPPORTED;
    std::vector<std::vector<void*>> peer_buf(P);
    std::vector<unsigned long long*> peer_sig(P, nullptr);   // mapped signal blocks (send and receive peers)
    auto open_sig = [&](int q) -> pepp_status_t {
        if (peer_sig[q]) return PEPP_OK;
        void* sig = nullptr;
        PEPP_CUDA_TRY(cudaIpcOpenMemHandle(&sig, all[q].sig, cudaIpcMemLazyEnablePeerAccess));
        p->p2p_opened.push_back(sig);
        peer_sig[q] = (unsigned long long*)sig;
        return PEPP_OK;
    };
    pepp_status_t s;
    for (size_t j = 0; j < sendp.size(); ++j) {
        const int q = sendp[j];
        peer_buf[q].assign(nbuf, nullptr);
        for (int b = 0; b < nbuf; ++b) {
            PEPP_CUDA_TRY(cudaIpcOpenMemHandle(&peer_buf[q][b], all[q].buf[b], cudaIpcMemLazyEnablePeerAccess));
            p->p2p_opened.push_back(peer_buf[q][b]);
        }
        if ((s = open_sig(q))) return s;
        p->p2p_ready_in[j] = p->d_sig + q;              // my ready[q]: q may now be written
        p->p2p_arrive_out[j] = peer_sig[q] + P + me;    // q's arrive[me]
    }
    for (size_t j = 0; j < recvp.size(); ++j) {
        const int q = recvp[j];
        if ((s = open_sig(q))) return s;
        p->p2p_ready_out[j] = peer_sig[q] + me;         // q's ready[me]: q may write into me
        p->p2p_arrive_in[j] = p->d_sig + P + q;         // my arrive[q]
    }
    p->p2p_nsend = (int)sendp.size();
    p->p2p_nrecv = (int)recvp.size();
    // push ranges: each peer's send range cut to the head and the tail segments
    const int64_t R = p->nrows, h = p->info.overlap_head, t = p->info.overlap_tail;
    int np = 0;
    for (auto& sr : p->send_rng) {
        for (int seg = 0; seg < 2; ++seg) {
            const int64_t lo = std::max(sr.lo, seg ? R - t : 0), hi = std::min(sr.hi, seg ? R : h);
            if (lo >= hi) continue;
            if (np == pepp::k::kP2PMaxPush) return PEPP_E_UNSUPPORTED;
            p->p2p_push_lo[np] = lo;
            p->p2p_push_hi[np] = hi;
            for (int b = 0; b < nbuf; ++b) p->p2p_push_dst[b][np] = peer_buf[sr.peer][b];
            ++np;
        }
    }
    p->p2p_npush = np;
    p->p2p_grid = (int)std::max<int64_t>(1, std::min<int64_t>((h + t + 255) / 256, 8 * kReserveSms));
    return PEPP_OK;
}

// Collective on every path: a rank whose export or import fails still takes
// part in the handle all-gather and the final agreement, so no peer is left
// waiting inside a collective; every rank returns an error if any failed.
pepp_status_t p2p_register(pepp_spmv_plan_t* p, int nbuf, cudaStream_t st) {
    const int P = p->opts.nranks, me = p->opts.rank;
    std::vector<P2PHandles> all(P);
    std::memset(all.data(), 0, sizeof(P2PHandles) * P);
    pepp_status_t s = p2p_export(p, nbuf, st, &all[me]);
    // all-gather the IPC handles (bytes) over the plan's communicator
    DevTmp<unsigned char> d_h;
    PEPP_CUDA_TRY(d_h.alloc(sizeof(P2PHandles) * P));
    PEPP_CUDA_TRY(cudaMemcpyAsync(d_h.p, all.data(), sizeof(P2PHandles) * P, cudaMemcpyHostToDevice, st));
    if (p->nccl->GroupStart()) return PEPP_E_NCCL;
    for (int r = 0; r < P; ++r) {
        unsigned char* at = d_h.p + sizeof(P2PHandles) * r;
        if (p->nccl->Broadcast(at, at, sizeof(P2PHandles), pepp::NCCL_INT8, r, p->comm, st)) { p->nccl->GroupEnd(); return PEPP_E_NCCL; }
    }
    if (p->nccl->GroupEnd()) return PEPP_E_NCCL;
    PEPP_CUDA_TRY(cudaMemcpyAsync(all.data(), d_h.p, sizeof(P2PHandles) * P, cudaMemcpyDeviceToHost, st));
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    bool all_ok = true;
    for (int r = 0; r < P; ++r) all_ok &= all[r].ok == 1;
    if (std::getenv("PEPP_DEBUG"))
        for (int r = 0; r < P; ++r)
            std::fprintf(stderr, "[pepp p2p] rank %d: slot %d ok=%lld first bytes %02x%02x%02x%02x local status %d\n", me, r,
                         (long long)all[r].ok, (unsigned char)all[r].sig.reserved[0], (unsigned char)all[r].sig.reserved[1],
                         (unsigned char)all[r].sig.reserved[2], (unsigned char)all[r].sig.reserved[3], (int)s);
    if (!s && all_ok) s = p2p_import(p, nbuf, all);
    else if (!s) { s = PEPP_E_CUDA; pepp::set_last_error("a peer rank could not export its buffers", "p2p_register", __LINE__); }
    if (const char* e = std::getenv("PEPP_P2P_TIMEOUT_MS")) p->p2p_timeout_ns = 1000000ull * (unsigned long long)std::atoll(e);
    // agreement (and the barrier after which pushes may start: every rank has
    // mapped its peers and zeroed its flags)
    int64_t fail = s ? 1 : 0;
    pepp_status_t sb = nccl_allmax(p, st, &fail);
    if (sb) return PEPP_E_NCCL;   // no agreement: the caller makes the plan's error sticky
    if (s) return s;              // agreed failure (every rank returns an error)
    if (fail) { pepp::set_last_error("a peer rank could not map its peers' buffers", "p2p_register", __LINE__); return PEPP_E_CUDA; }
    p->p2p_nbuf = nbuf;
    return PEPP_OK;
}

template <typename T>
pepp_status_t p2p_launch_t(pepp_spmv_plan_t* p, int b, const T* x, T* y, cudaStream_t st) {
    pepp::k::P2PArgs<T> a{};
    const int64_t R = p->nrows, h = p->info.overlap_head, t = p->info.overlap_tail;
    a.seg_lo[0] = 0; a.seg_hi[0] = h;
    a.seg_lo[1] = R - t; a.seg_hi[1] = R;
    a.row_offset = p->row_offset;
    a.npush = p->p2p_npush;
    for (int j = 0; j < a.npush; ++j) {
        a.push_lo[j] = p->p2p_push_lo[j];
        a.push_hi[j] = p->p2p_push_hi[j];
        a.push_dst[j] = (T*)p->p2p_push_dst[b][j];
    }
    a.nsend = p->p2p_nsend;
    for (int j = 0; j < a.nsend; ++j) {
        a.ready_in[j] = p->p2p_ready_in[j];
        a.arrive_out[j] = p->p2p_arrive_out[j];
    }
    a.nrecv = p->p2p_nrecv;
    for (int j = 0; j < a.nrecv; ++j) {
        a.ready_out[j] = p->p2p_ready_out[j];
        a.arrive_in[j] = p->p2p_arrive_in[j];
    }
    const int P = p->opts.nranks;
    a.epoch = p->d_sig + 2 * P;
    a.done = (unsigned int*)(p->d_sig + 2 * P + 1);
    a.err = p->d_err;
    a.timeout_ns = p->p2p_timeout_ns;
    pepp::k::halo_push_kernel<T><<<p->p2p_grid, 256, 0, st>>>(p->d_rp, p->d_col, (const T*)p->d_val, x, y, a);
    return cudaGetLastError() == cudaSuccess ? PEPP_OK : PEPP_E_CUDA;
}

// a rank can run the fused push when the rows it sends lie in its head /
// tail split (sub-plans) or when it sends nothing (it then only signals)
bool p2p_capable(const pepp_spmv_plan_t* p) {
    if (p->sub[1]) return true;
    for (const auto& t : p->send_x) if (t.count) return false;
    return true;
}

// index of the registered buffer y points to, -1 if none
int p2p_index(const pepp_spmv_plan_t* p, const void* y) {
    for (int b = 0; b < p->p2p_nbuf; ++b) if (p->p2p_buf[b] == y) return b;
    return -1;
}

pepp_status_t plan_impl(const pepp_csr_t* A, const pepp_spmv_opts_t* o, pepp_spmv_plan_t* p) {
    // ---- argument checks (host, O(1)) ----
    if (A->nrows < 0 || A->ncols < 0 || A->nnz < 0 || !A->row_ptr) return PEPP_E_INVALID;
    if (A->nnz > 0 && (!A->col_idx || !A->values)) return PEPP_E_INVALID;
    if (A->value_type != PEPP_VALUE_F64 && A->value_type != PEPP_VALUE_F32) return PEPP_E_INVALID;
    p->vt = A->value_type;
    p->esz = p->vt == PEPP_VALUE_F32 ? sizeof(float) : sizeof(double);
    if (o->nranks < 1 || o->rank < 0 || o->rank >= o->nranks) return PEPP_E_INVALID;
    if (o->nranks > 1 && !o->row_bounds) return PEPP_E_INVALID;
    if (A->nnz + 8 >= (int64_t)INT32_MAX || A->ncols >= (int64_t)INT32_MAX || A->nrows >= (int64_t)INT32_MAX)
        return PEPP_E_UNSUPPORTED;
    if (o->variant_mask != 0 && (o->variant_mask & ((1u << PEPP_V_COUNT) - 1)) == 0) return PEPP_E_INVALID;

    p->opts = *o;
#ifdef PEPP_EXP_RESERVE_SMS   // experiments only (tools/overlap_cost.py): SMs a top-level plan's persistent grids leave free
    if (!p->reserve_sms) p->reserve_sms = PEPP_EXP_RESERVE_SMS;
#endif
    p->nrows = A->nrows; p->ncols = A->ncols; p->nnz = A->nnz; p->first = A->first;
    p->pad = (int)(((A->first % 4) + 4) % 4);
    if (o->nranks > 1) {
        p->row_bounds.assign(o->row_bounds, o->row_bounds + o->nranks + 1);
        for (int r = 0; r < o->nranks; ++r) if (p->row_bounds[r + 1] < p->row_bounds[r]) return PEPP_E_INVALID;
        if (p->row_bounds[o->rank + 1] - p->row_bounds[o->rank] != A->nrows) return PEPP_E_INVALID;
        p->row_offset = p->row_bounds[o->rank];
        p->global_rows = p->row_bounds[o->nranks];
    } else {
        p->row_bounds = {0, A->nrows};
        p->row_offset = 0;
        p->global_rows = A->nrows;
    }
    if (o->history_path) p->history_path = o->history_path;
    p->opts.history_path = nullptr;   // borrowed pointers are not kept past this call
    p->opts.row_bounds = nullptr;

    // ---- device ----
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) { (void)cudaGetLastError(); return PEPP_E_CUDA; }
    if (o->device >= 0) { if (o->device >= ndev) return PEPP_E_INVALID; p->device = o->device; }
    else PEPP_CUDA_TRY(cudaGetDevice(&p->device));
    PEPP_CUDA_TRY(cudaSetDevice(p->device));
    PEPP_CUDA_TRY(cudaDeviceGetAttribute(&p->sm_count, cudaDevAttrMultiProcessorCount, p->device));
    cudaStream_t st = nullptr;
    PEPP_CUDA_TRY(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    struct StreamGuard { cudaStream_t s; ~StreamGuard() { cudaStreamDestroy(s); } } guard{st};

    // row_ptr[0] == first (A1) is checked on the host (one value)
    int64_t rp0 = 0, rpn = 0;
    if (A->on_device) {
        PEPP_CUDA_TRY(cudaMemcpy(&rp0, A->row_ptr, sizeof(int64_t), cudaMemcpyDeviceToHost));
        PEPP_CUDA_TRY(cudaMemcpy(&rpn, A->row_ptr + A->nrows, sizeof(int64_t), cudaMemcpyDeviceToHost));
    } else {
        rp0 = A->row_ptr[0];
        rpn = A->row_ptr[A->nrows];
    }
    if (rp0 != A->first || rpn - A->first != A->nnz) return PEPP_E_INVALID;

    // ---- a1: copy + narrow row_ptr, validate, context statistics ----
    pepp_status_t s;
    const int64_t nstore = p->pad + A->nnz + 8;   // + trailing zeros for aligned 4-groups
    if ((s = dalloc(p, &p->d_rp, A->nrows + 1 + 8))) return s;   // +8: aligned 16-B bulk copies may overrun
    PEPP_CUDA_TRY(cudaMemsetAsync(p->d_rp, 0, sizeof(int) * (A->nrows + 1 + 8), st));
    if ((s = dalloc(p, &p->d_col, nstore))) return s;
    if ((s = dalloc_bytes(p, &p->d_val, nstore * (int64_t)p->esz))) return s;
    PEPP_CUDA_TRY(cudaMemsetAsync(p->d_col, 0, sizeof(int) * nstore, st));
    PEPP_CUDA_TRY(cudaMemsetAsync(p->d_val, 0, p->esz * nstore, st));
    const cudaMemcpyKind kind = A->on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    if (A->nnz) {
        if ((s = upload(p->d_col + p->pad, A->col_idx, sizeof(int) * A->nnz, kind, st))) return s;
        if ((s = upload((char*)p->d_val + p->pad * p->esz, A->values, p->esz * A->nnz, kind, st))) return s;
    }
    DevTmp<int64_t> rp64;
    DevTmp<pepp::k::RowStats> stats;
    PEPP_CUDA_TRY(rp64.alloc(A->nrows + 1));
    PEPP_CUDA_TRY(stats.alloc(1));
    int64_t* d_rp64 = rp64.p;
    pepp::k::RowStats* d_stats = stats.p;
    PEPP_CUDA_TRY(cudaMemsetAsync(d_stats, 0, sizeof(pepp::k::RowStats), st));
    if ((s = upload(d_rp64, A->row_ptr, sizeof(int64_t) * (A->nrows + 1), kind, st))) return s;
    {
        const int tb = 256;
        const int gb = (int)std::min<int64_t>((A->nrows + 1 + tb - 1) / tb, (int64_t)p->sm_count * 8);
        pepp::k::rowptr_check_narrow_kernel<<<gb, tb, 0, st>>>(A->nrows, d_rp64, A->first, p->pad, p->d_rp, d_stats);
        PEPP_CUDA_TRY(cudaGetLastError());
        if (o->validate && A->nnz) {
            const int gc = (int)std::min<int64_t>((A->nnz + tb - 1) / tb, (int64_t)p->sm_count * 8);
            pepp::k::col_check_kernel<<<gc, tb, 0, st>>>(A->nnz, p->d_col + p->pad, A->ncols, &d_stats->bad);
            PEPP_CUDA_TRY(cudaGetLastError());
        }
    }
    pepp::k::RowStats hs{};
    PEPP_CUDA_TRY(cudaMemcpyAsync(&hs, d_stats, sizeof(hs), cudaMemcpyDeviceToHost, st));
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    std::vector<int32_t> ghosts;
    if (o->nranks > 1) {
        std::vector<int32_t> hcol(A->nnz);
        if (A->nnz) PEPP_CUDA_TRY(cudaMemcpy(hcol.data(), p->d_col + p->pad, sizeof(int) * A->nnz, cudaMemcpyDeviceToHost));
        pepp::halo_ghost_list(hcol.data(), A->nnz, p->row_offset, p->row_offset + A->nrows, ghosts);
        if (!ghosts.empty() && (ghosts.front() < 0 || ghosts.back() >= p->global_rows)) hs.bad = 1;
    }
    if (hs.bad) return PEPP_E_INVALID;

    pepp_plan_info_t& I = p->info;
    I.nrows = A->nrows; I.ncols = A->ncols; I.nnz = A->nnz;
    I.mean_row = A->nrows ? (double)A->nnz / (double)A->nrows : 0.0;
    {
        const double m = I.mean_row;
        const double ex2 = A->nrows ? (double)hs.sum_len2_lo / (double)A->nrows : 0.0;
        const double var = std::max(0.0, ex2 - m * m);
        I.cv_row = m > 0 ? std::sqrt(var) / m : 0.0;
    }
    I.max_row = (int64_t)hs.max_len;
    I.empty_rows = (int64_t)hs.empty;
    I.nranks = o->nranks; I.rank = o->rank; I.row_offset = p->row_offset;
    I.algorithmic_bytes = A->nnz * 12 + (A->nrows + 1) * 4 + A->ncols * 8 + A->nrows * 8;

    // ---- a3: candidates + variant preparation ----
    // multi-stage composition (P@10489): static narrowing from the context
    // instance, then the runtime's history-based choice among the rest
    uint32_t mask = o->variant_mask ? o->variant_mask : 0xffffffffu;
    if (o->prune) {
        const double mean = I.mean_row;
        uint32_t keep = mask;
        if ((double)I.max_row > std::max(4096.0, 256.0 * mean)) keep &= ~(1u << PEPP_V_CSR_VECTOR);

        if (keep & ((1u << PEPP_V_COUNT) - 1)) mask = keep;   // never prune everything
    }
    if (mask & (1u << PEPP_V_CSR_VECTOR))
        for (int tpr : {2, 4, 8, 16, 32}) p->cands.push_back({PEPP_V_CSR_VECTOR, tpr});
    if (mask & (1u << PEPP_V_MERGE_PATH)) {
        p->cands.push_back({PEPP_V_MERGE_PATH, kMergeIPT});
        p->cands.push_back({PEPP_V_MERGE_PATH, kMergeWarpParam});
    }
    // (SELL chunk lengths stay below kSellLenMask: rows above the hybrid cap leave the layout)
    if ((mask & ((1u << PEPP_V_COUNT) - 1)) == 0) return PEPP_E_UNSUPPORTED;
    if (mask & (1u << PEPP_V_SELL)) {
        if ((s = prepare_sell(p, st))) return s;
        p->cands.push_back({PEPP_V_SELL, p->sell_sigma});
    }
    if (mask & (1u << PEPP_V_MERGE_PATH)) { if ((s = prepare_merge(p, st))) return s; }
    if (mask & (1u << PEPP_V_CSR_STREAM)) {
        if ((s = prepare_stream(p, st))) return s;
        p->cands.push_back({PEPP_V_CSR_STREAM, kStreamNB});
    }
    if (mask & (1u << PEPP_V_PANEL)) {   // only where x is far beyond L2 and rows reach across it
        std::vector<int> lgs;
        if ((s = prepare_panels(p, st, &lgs))) return s;
        for (int lg : lgs) p->cands.push_back({PEPP_V_PANEL, lg});
    }
    if (p->cands.empty()) return PEPP_E_UNSUPPORTED;
    p->eligible.assign(p->cands.size(), 1);
    p->pending.assign(p->cands.size(), 0);
    p->warmed.assign(p->cands.size(), 0);
    {   // bytes each candidate moves per call (pepp_choice_t.layout_bytes)
        const int64_t es = (int64_t)p->esz;
        const int64_t csr = A->nnz * (es + 4) + (A->nrows + 1) * 4 + A->ncols * es + A->nrows * es;
        for (const Candidate& c : p->cands) {
            int64_t b = csr;
            if (c.variant == PEPP_V_SELL) b = p->sell_bytes;
            else if (c.variant == PEPP_V_MERGE_PATH) {
                const int64_t nt = c.param == kMergeWarpParam ? p->ntiles_w : p->ntiles;
                b += (nt + 1) * 8 + nt * 2 * (4 + 8);   // tile coordinates, carries written and read back
            } else if (c.variant == PEPP_V_CSR_STREAM) {
                b += (int64_t)p->nitems * 16 + (int64_t)p->nlong * 16;
            } else if (c.variant == PEPP_V_PANEL) {
                // entries (column + value), pairs (row + start), y zeroed then
                // read and written once per pair, x read once
                int64_t np = 0;
                for (const auto& pl : p->panels) if (pl.lg == c.param) np = pl.npairs;
                b = A->nnz * (es + 4) + np * (8 + 2 * es) + A->nrows * es + A->ncols * es;
            }
            p->cand_bytes.push_back(b);
        }
    }
    I.ncandidates = (int32_t)p->cands.size();

    p->grid_csr[1] = grid_for((const void*)pepp::k::csr_vector_kernel<2, kBlock, double>, kBlock, A->nrows, kBlock / 2, p->sm_count);
    p->grid_csr[2] = grid_for((const void*)pepp::k::csr_vector_kernel<4, kBlock, double>, kBlock, A->nrows, kBlock / 4, p->sm_count);
    p->grid_csr[3] = grid_for((const void*)pepp::k::csr_vector_kernel<8, kBlock, double>, kBlock, A->nrows, kBlock / 8, p->sm_count);
    p->grid_csr[4] = grid_for((const void*)pepp::k::csr_vector_kernel<16, kBlock, double>, kBlock, A->nrows, kBlock / 16, p->sm_count);
    p->grid_csr[5] = grid_for((const void*)pepp::k::csr_vector_kernel<32, kBlock, double>, kBlock, A->nrows, kBlock / 32, p->sm_count);
    {   // SELL: exactly one resident wave; warps walk their chunks with prefetch
        int occ = 0;
        const bool srt = p->d_perm != nullptr, pat = p->sell_const_chunks > 0, f32 = p->vt == PEPP_VALUE_F32;
        const void* fn = f32 ? (srt ? (pat ? (const void*)pepp::k::sell_kernel<kBlock, true, true, float> : (const void*)pepp::k::sell_kernel<kBlock, true, false, float>)
                                    : (pat ? (const void*)pepp::k::sell_kernel<kBlock, false, true, float> : (const void*)pepp::k::sell_kernel<kBlock, false, false, float>))
                             : (srt ? (pat ? (const void*)pepp::k::sell_kernel<kBlock, true, true, double> : (const void*)pepp::k::sell_kernel<kBlock, true, false, double>)
                                    : (pat ? (const void*)pepp::k::sell_kernel<kBlock, false, true, double> : (const void*)pepp::k::sell_kernel<kBlock, false, false, double>));
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, kBlock, 0) != cudaSuccess || occ < 1) occ = 1;
        (void)cudaGetLastError();
        const int64_t need = ((int64_t)p->nchunks + kBlock / 32 - 1) / (kBlock / 32);
        const int64_t wave = (int64_t)std::max(1, p->sm_count - p->reserve_sms) * occ;
        // prefetching pays once a warp walks many chunks; small matrices keep
        // more (shorter-lived) blocks instead
        const int64_t cap = need >= 16 * wave ? wave : 4 * wave;
        p->grid_sell = (int)std::max<int64_t>(1, std::min<int64_t>(need, cap));
        if (p->d_perm && (s = sell_warp_ranges(p))) return s;
        if (!p->d_perm && p->d_patlist && kPatInterleave && (s = sell_patlist_interleave(p))) return s;
    }

    // ---- history ----
    // the instance bits keep fp32 / value-compressed plans (different kernels,
    // ~1.6x apart on config 4) from sharing history records with fp64 ones
    p->key = pepp::context_key(A->nrows, A->ncols, A->nnz, I.cv_row, o->nranks,
                               (p->vt == PEPP_VALUE_F32 ? PEPP_KEY_F32 : 0) | (o->compress_values ? PEPP_KEY_COMPRESS : 0));
    I.key = p->key;
    p->hist = pepp::history_new();
    if (!p->hist) return PEPP_E_NOMEM;
    if (!p->history_path.empty()) (void)pepp_history_load(p->hist, p->history_path.c_str());
    {
        const int32_t n = (int32_t)p->cands.size();
        p->uids.resize(n);
        for (int32_t c = 0; c < n; ++c) p->uids[c] = (p->cands[c].variant << 20) | (p->cands[c].param & 0xFFFFF);
        p->prior.assign(n, -1.0);
        p->order.resize(n);
        for (int32_t c = 0; c < n; ++c) p->order[c] = c;
        bool have_prior = n && pepp::history_prior(p->hist, p->key, n, p->uids.data(), p->prior.data(), &p->prior_key);
        if (have_prior) p->info.prior_key = p->prior_key;
        if (o->predict) {   // the descriptor's prediction function (M6, P@6887)
            p->predicted.assign(n, -1.0);
            for (int32_t c = 0; c < n; ++c) {
                const double v = o->predict(&p->info, p->cands[c].variant, p->cands[c].param, o->predict_user);
                if (v > 0 && std::isfinite(v)) { p->predicted[c] = v; ++p->info.predicted; }
            }
            if (!have_prior && p->info.predicted) { p->prior = p->predicted; have_prior = true; }
        }
        if (have_prior) {
            // a recorded neighbour context orders the calibration by its means;
            // a *variant* it never recorded at all (e.g. the column panels,
            // which only exist once x leaves L2, so a smaller neighbour cannot
            // have timed them) is tried first — optimism under uncertainty: its
            // one calibration call costs less than missing a new best variant
            // (round-2 sweep: cold picks 2.15x / 2.35x off on the two largest
            // random matrices without it). Predictions keep their own order.
            std::vector<uint8_t> unseen(n, 0);
            if (p->prior_key) {
                for (int32_t c = 0; c < n; ++c) {
                    bool seen = false;
                    for (int32_t d = 0; d < n && !seen; ++d) seen = p->cands[d].variant == p->cands[c].variant && p->prior[d] > 0;
                    unseen[c] = !seen;
                }
            }
            std::stable_sort(p->order.begin(), p->order.end(), [&](int32_t a, int32_t b) {
                const double pa = unseen[a] ? 0.0 : p->prior[a] > 0 ? p->prior[a] : 1e300;
                const double pb = unseen[b] ? 0.0 : p->prior[b] > 0 ? p->prior[b] : 1e300;
                return pa < pb;
            });
        }
    }
    for (auto& r : p->ring) {
        PEPP_CUDA_TRY(cudaEventCreate(&r.start));
        PEPP_CUDA_TRY(cudaEventCreate(&r.stop));
    }

    // ---- a2: exchange setup (partitioned calls) ----
    p->exchange = PEPP_X_NONE;
    if (o->nranks > 1) {
        p->nccl = pepp::nccl_load();
        if (!p->nccl) return PEPP_E_NCCL;
        if (o->nccl_comm) {
            p->comm = (ncclComm_t)o->nccl_comm;
        } else {
            if (!o->nccl_unique_id) return PEPP_E_INVALID;
            pepp::ncclUniqueId id;
            std::memcpy(&id, o->nccl_unique_id, sizeof(id));
            if (p->nccl->CommInitRank(&p->comm, o->nranks, id, o->rank)) return PEPP_E_NCCL;
            p->own_comm = true;
        }
        p->opts.nccl_unique_id = nullptr;
        if ((s = setup_halo(p, ghosts, st))) return s;
        int ex = o->exchange;
        if (ex == PEPP_X_AUTO) {
            // halo when every rank's ghosts are a small part of x;
            // the decision must be identical on all ranks: max-reduce the counts.
            DevTmp<int64_t> d_g;
            int64_t g = (int64_t)ghosts.size(), gmax = 0;
            PEPP_CUDA_TRY(d_g.alloc(1));
            PEPP_CUDA_TRY(cudaMemcpy(d_g.p, &g, sizeof(int64_t), cudaMemcpyHostToDevice));
            if (p->nccl->AllReduce(d_g.p, d_g.p, 1, pepp::NCCL_INT64, pepp::NCCL_OP_MAX, p->comm, st)) return PEPP_E_NCCL;
            PEPP_CUDA_TRY(cudaStreamSynchronize(st));
            PEPP_CUDA_TRY(cudaMemcpy(&gmax, d_g.p, sizeof(int64_t), cudaMemcpyDeviceToHost));
            ex = ((double)gmax < 0.25 * (double)p->global_rows) ? PEPP_X_HALO : PEPP_X_ALLGATHER;
        }
        p->exchange = ex;
    }
    I.exchange = p->exchange;
    if (p->exchange == PEPP_X_HALO && o->overlap && !p->send_local.empty())
        if ((s = setup_overlap(A, o, p))) return s;
    p->send_local.clear();
    p->send_local.shrink_to_fit();
    // distribution candidates (P' < nranks) for the plan-time timing (dist_probe)
    if (o->nranks > 1 && o->dist_select && o->use_history && p->ncols == p->global_rows)
        if ((s = setup_dist_parts(o, p, ghosts, st))) return s;
    I.device_bytes = p->dev_bytes;
    for (auto* q : p->sub) if (q) I.device_bytes += q->dev_bytes;
    for (auto& dp : p->dparts) if (dp.plan) I.device_bytes += dp.plan->dev_bytes;
    return PEPP_OK;
}

pepp_status_t dist_probe(pepp_spmv_plan_t* p);

}  // namespace

// ================================================================= C-ABI
extern "C" PEPP_API pepp_status_t pepp_spmv_exec(pepp_spmv_plan_t* p, const void* x, void* y, int flags,
                                                void* stream, const pepp_choice_t* force, pepp_choice_t* used);

namespace {
// Per-plan device scratch — merge-path / CSR-stream carries, hybrid-SELL
// partial sums and row counters, halo pack buffers and the side stream — is
// shared by all of the plan's calls. Calls on one stream are ordered by the
// stream; a call that uses scratch on another stream than the previous user
// first waits for that user (an event), so two in-flight calls never
// interleave on it. Scratch-free candidates (vector-CSR, SELL without long
// rows, no exchange) skip this and keep overlapping across streams (inter-
// call parallelism, §IV-E P@21908–27091). Not applied under graph capture:
// a captured call's ordering is the graph's.
bool uses_scratch(const pepp_spmv_plan_t* p, const Candidate& c) {
    if (c.variant == PEPP_V_MERGE_PATH || c.variant == PEPP_V_CSR_STREAM) return true;
    return c.variant == PEPP_V_SELL && p->nsell_seg > 0;
}

pepp_status_t scratch_acquire(pepp_spmv_plan_t* p, cudaStream_t st) {
    if (!p->ev_scratch) PEPP_CUDA_TRY(cudaEventCreateWithFlags(&p->ev_scratch, cudaEventDisableTiming));
    if (p->scratch_used && p->scratch_stream != st) PEPP_CUDA_TRY(cudaStreamWaitEvent(st, p->ev_scratch, 0));
    return PEPP_OK;
}

pepp_status_t scratch_release(pepp_spmv_plan_t* p, cudaStream_t st) {
    PEPP_CUDA_TRY(cudaEventRecord(p->ev_scratch, st));
    p->scratch_stream = st;
    p->scratch_used = true;
    return PEPP_OK;
}

// The interior rows compute on the caller's stream while a high-priority side
// stream computes the head and tail rows (into the SMs the interior's
// persistent grid leaves free) and then runs the halo exchange, which reads
// only head / tail rows and writes only other ranks' rows of y; the caller's
// stream joins the side stream. Critical path: max(interior, head + tail +
// exchange) instead of kernel + exchange.
pepp_status_t exec_overlap(pepp_spmv_plan_t* p, const void* x, void* y, int flags, cudaStream_t st,
                           pepp_choice_t* used, bool allow_p2p) {
    char* yb = (char*)y + p->row_offset * (int64_t)p->esz;
    const int sf = flags & PEPP_EXEC_NO_TIMING;
    // the side stream starts after everything the caller queued (x is ready)
    PEPP_CUDA_TRY(cudaEventRecord(p->ev_fork, st));
    PEPP_CUDA_TRY(cudaStreamWaitEvent(p->side, p->ev_fork, 0));
    // interior first (the host may block inside a synchronous exchange)
    pepp_choice_t u{};
    // a rank that sends nothing (no split) computes its whole block as the
    // "interior" through its own selection (PEPP_Y_LOCAL: no exchange)
    pepp_status_t s = p->sub[1] ? pepp_spmv_exec(p->sub[1], x, yb + p->sub_r0[1] * (int64_t)p->esz, sf, st, nullptr, &u)
                                : pepp_spmv_exec(p, x, y, sf | PEPP_Y_LOCAL, st, nullptr, &u);
    const int b = allow_p2p ? p2p_index(p, y) : -1;
    if (b >= 0) {
        // fused: head + tail rows computed, pushed into the peers' buffer b and
        // signalled by one kernel (PEPP_X_P2P)
        if (!s) s = p->vt == PEPP_VALUE_F32 ? p2p_launch_t<float>(p, b, (const float*)x, (float*)y, p->side)
                                            : p2p_launch_t<double>(p, b, (const double*)x, (double*)y, p->side);
        u.launches += 1;
    } else {
        for (int i : {0, 2})
            if (!s && p->sub[i]) {
                pepp_choice_t ui{};
                s = pepp_spmv_exec(p->sub[i], x, yb + p->sub_r0[i] * (int64_t)p->esz, sf, p->side, nullptr, &ui);
                u.launches += ui.launches;
            }
        if (!s) s = exchange_halo(p, y, p->side);
        u.launches += halo_kernels(p);
    }
    PEPP_CUDA_TRY(cudaEventRecord(p->ev_join, p->side));   // join whatever reached the side stream
    PEPP_CUDA_TRY(cudaStreamWaitEvent(st, p->ev_join, 0));
    if (s) return s;
    u.nparts = p->opts.nranks;
    u.exchange = b >= 0 ? PEPP_X_P2P : PEPP_X_HALO;
    if (used) *used = u;
    return PEPP_OK;
}

// One call under a distribution candidate with P' < nranks: ranks 0..P'-1
// compute their P' block (its own history-based variant selection), then
// the exchange: the P' blocks all-gathered to every rank (PEPP_X_ALLGATHER,
// or any PEPP_Y_REPLICATED call), or (PEPP_X_HALO) the halo among the P'
// ranks followed by every rank receiving its own rows and own ghosts from
// their P' owners — so the call leaves y as a P' = nranks call would for
// this rank's own block (own rows + the entries its next call reads).
pepp_status_t exec_dist(pepp_spmv_plan_t* p, DistPart& dp, int ex, const void* x, void* y, int flags, cudaStream_t st,
                        const pepp_choice_t* force, pepp_choice_t* used) {
    pepp_choice_t u{};
    pepp_status_t s = PEPP_OK;
    if (dp.plan) {
        pepp_choice_t f{};
        const pepp_choice_t* fp = nullptr;
        if (force && force->variant >= 0) { f = *force; f.nparts = 0; f.exchange = PEPP_X_AUTO; fp = &f; }
        s = pepp_spmv_exec(dp.plan, x, y, flags & PEPP_EXEC_NO_TIMING, st, fp, &u);
        if (s) return s;
    }
    if ((flags & PEPP_Y_REPLICATED) || ex == PEPP_X_ALLGATHER) {
        ex = PEPP_X_ALLGATHER;
        s = exchange_blocks(p, dp.bounds.data(), dp.parts, y, st);
    } else {
        if (dp.plan && dp.parts > 1) {
            s = exchange_halo(dp.plan, y, st);
            u.launches += halo_kernels(dp.plan);
        }
        if (!s) s = exchange_xfer(p, dp.recv_x, dp.send_x, y, st);
        u.launches += xfer_kernels(dp.recv_x, dp.send_x);
        if (!s) s = dist_complete(p, y, st, dp.parts, &u.launches);
    }
    if (s) return s;
    u.nparts = dp.parts;
    u.exchange = ex;
    if (used) *used = u;
    return PEPP_OK;
}

// the plans whose kernels a distribution candidate runs on this rank are
// still calibrating their variant choice (so the candidate is not timed yet)
bool dist_busy(const pepp_spmv_plan_t* p, int parts, int ex) {
    auto busy = [](const pepp_spmv_plan_t* q) { return q && q->opts.use_history && !q->calibrated && q->cands.size() > 1; };
    if (parts == p->opts.nranks) {
        if (ex == PEPP_X_HALO && p->sub[1]) return busy(p->sub[0]) || busy(p->sub[1]) || busy(p->sub[2]);
        return busy(p);
    }
    for (const auto& dp : p->dparts) if (dp.parts == parts) return busy(dp.plan);
    return false;
}
}  // namespace

extern "C" PEPP_API pepp_status_t pepp_spmv_plan(const pepp_csr_t* A, const pepp_spmv_opts_t* opts,
                                                pepp_spmv_plan_t** out) {
    PEPP_NVTX("pepp_spmv_plan");
    if (!out) return PEPP_E_INVALID;
    *out = nullptr;
    if (!A) return PEPP_E_INVALID;
    pepp_spmv_opts_t def;
    pepp_spmv_opts_default(&def);
    if (!opts) opts = &def;
    pepp_spmv_plan_t* p = new (std::nothrow) pepp_spmv_plan_t();
    if (!p) return PEPP_E_NOMEM;
    p->device = -1;
    int caller_dev = -1;
    if (cudaGetDevice(&caller_dev) != cudaSuccess) { (void)cudaGetLastError(); caller_dev = -1; }
    struct Restore { int d; ~Restore() { if (d >= 0) cudaSetDevice(d); (void)cudaGetLastError(); } } restore{caller_dev};
    pepp_status_t s;
    try {
        s = plan_impl(A, opts, p);
    } catch (const std::bad_alloc&) {
        s = PEPP_E_NOMEM;
    } catch (...) {
        s = PEPP_E_INVALID;
    }
    // P and exchange as timed choices: every candidate timed, ranks agree
    if (s == PEPP_OK && p->opts.nranks > 1 && p->opts.dist_select && p->opts.use_history && p->ncols == p->global_rows) {
        try {
            s = dist_probe(p);
        } catch (const std::bad_alloc&) {
            s = PEPP_E_NOMEM;
        }
    }
    if (s != PEPP_OK) { free_plan(p); return s; }
    *out = p;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_select(pepp_spmv_plan_t* p, pepp_choice_t* out) {
    if (!p || !out) return PEPP_E_INVALID;
    if (p->sticky) return p->sticky;
    const pepp_status_t s = select_choice(p, out);
    if (!s && p->dist_next >= 0) {   // partitioned: the distribution a PEPP_Y_NEXT_INPUT call runs
        out->nparts = p->info.dist_nparts;
        out->exchange = p->info.dist_exchange;
    }
    return s;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_exec(pepp_spmv_plan_t* p, const void* x, void* y, int flags,
                                                void* stream, const pepp_choice_t* force, pepp_choice_t* used) {
    PEPP_NVTX("pepp_spmv_exec");
    if (!p) return PEPP_E_INVALID;
    if (p->sticky) return p->sticky;
    if ((!x && p->ncols > 0) || (!y && p->global_rows > 0)) return PEPP_E_INVALID;
    if (x && y) {   // x [0, ncols) and y [0, global_rows) must not overlap
        const char *xb = (const char*)x, *xe = xb + p->ncols * (int64_t)p->esz;
        const char *yb = (const char*)y, *ye = yb + p->global_rows * (int64_t)p->esz;
        if (xb < ye && yb < xe) return PEPP_E_INVALID;
    }
    if (p->h_err && *(volatile int*)p->h_err) return p->sticky = PEPP_E_NCCL;   // a peer never arrived (P2P)
    cudaStream_t st = (cudaStream_t)stream;
    DeviceScope dscope(p->device);
    if (!dscope.ok) return PEPP_E_CUDA;
    bool capturing = false;
    {
        cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
        if (cudaStreamIsCapturing(st, &cs) != cudaSuccess) { (void)cudaGetLastError(); cs = cudaStreamCaptureStatusNone; }
        capturing = cs != cudaStreamCaptureStatusNone;
    }
    // ---- partitioned calls: the distribution (P', exchange) of this call
    const int N = p->opts.nranks;
    const bool fvar = force && force->variant >= 0;   // variant forced (PEPP_V_AUTO = selected as usual)
    const bool part_call = N > 1 && (flags & (PEPP_Y_NEXT_INPUT | PEPP_Y_REPLICATED));
    const bool next_only = (flags & PEPP_Y_NEXT_INPUT) && !(flags & PEPP_Y_REPLICATED);
    int ex_call = p->exchange;                        // exchange of a P' = nranks call
    bool allow_p2p = p->dcands.empty() || p->p2p_use;
    DistPart* dpart = nullptr;
    if (part_call) {
        if (force && force->nparts > 0 && force->nparts != N) {   // a forced P' < nranks
            for (auto& dp : p->dparts) if (dp.parts == force->nparts) dpart = &dp;
            if (!dpart) return PEPP_E_INVALID;
            ex_call = force->exchange == PEPP_X_ALLGATHER ? PEPP_X_ALLGATHER : PEPP_X_HALO;
        } else if (force && (force->exchange == PEPP_X_ALLGATHER || force->exchange == PEPP_X_HALO)) {
            ex_call = force->exchange;
            allow_p2p = false;
        } else if (force && force->exchange == PEPP_X_P2P) {
            allow_p2p = true;
        } else if (!force && !p->dcands.empty() && !(next_only && allow_p2p && p2p_index(p, y) >= 0)) {
            // the distribution the plan-time timing chose (opts.dist_select)
            const int d = (flags & PEPP_Y_REPLICATED) ? p->dist_repl : p->dist_next;
            if (d >= 0) {
                if (p->dcands[d].parts != N)
                    for (auto& dp : p->dparts) if (dp.parts == p->dcands[d].parts) dpart = &dp;
                ex_call = p->dcands[d].ex;
            }
            allow_p2p = false;
        }
    }
    if (dpart) {
        pepp_status_t s = capturing ? PEPP_OK : scratch_acquire(p, st);
        if (!s) s = exec_dist(p, *dpart, ex_call, x, y, flags, st, force, used);
        if (!s && !capturing) s = scratch_release(p, st);
        if (s) p->sticky = s;
        else ++p->ncalls;
        return s;
    }
    if (!fvar && next_only && ex_call == PEPP_X_HALO && (p->sub[1] || (allow_p2p && p2p_index(p, y) >= 0))) {
        pepp_status_t s = capturing ? PEPP_OK : scratch_acquire(p, st);
        if (!s) s = exec_overlap(p, x, y, flags, st, used, allow_p2p);
        if (!s) s = dist_complete(p, y, st, N, used ? &used->launches : nullptr);
        if (!s && !capturing) s = scratch_release(p, st);
        if (s) p->sticky = s;
        else ++p->ncalls;
        return s;
    }
    pepp_choice_t ch{};
    if (fvar) {
        int idx = -1;
        for (size_t i = 0; i < p->cands.size(); ++i)
            if (p->cands[i].variant == force->variant && (force->param <= 0 || p->cands[i].param == force->param)) { idx = (int)i; break; }
        if (idx < 0) return PEPP_E_INVALID;
        fill_choice(p, idx, 0, 0.0, &ch);
        if (!capturing) harvest(p, false);
    } else {
        pepp_status_t s = select_choice(p, &ch, capturing);
        if (s) return s;
    }

    // scratch ordering first: a wait for another stream is not the call's time
    const bool exchanging = p->opts.nranks > 1 && (flags & (PEPP_Y_NEXT_INPUT | PEPP_Y_REPLICATED));
    const bool scr = !capturing && (exchanging || uses_scratch(p, p->cands[ch.candidate]));
    if (scr) {
        pepp_status_t s = scratch_acquire(p, st);
        if (s) { p->sticky = s; return s; }
    }
    // timing: every calibration call and every forced call, then every
    // sample_period-th call; never inside a CUDA graph capture
    bool timed = !(flags & PEPP_EXEC_NO_TIMING) && !capturing;
    if (timed && !force && !ch.calibrating)
        timed = p->opts.sample_period > 0 && (p->ncalls % p->opts.sample_period) == 0;
    if (timed && p->ring_count == kTimingRing) timed = false;
    TimingRec* rec = nullptr;
    if (timed) {
        rec = &p->ring[(p->ring_head + p->ring_count) % kTimingRing];
        if (cudaEventRecord(rec->start, st) != cudaSuccess) { (void)cudaGetLastError(); rec = nullptr; }
    }
    pepp_status_t s = launch(p, p->cands[ch.candidate], x, (char*)y + p->row_offset * (int64_t)p->esz, st);
    if (s) { p->sticky = s; return s; }
    ch.launches = launches_for(p, p->cands[ch.candidate], x, (char*)y + p->row_offset * (int64_t)p->esz);
    if (rec) {
        if (cudaEventRecord(rec->stop, st) == cudaSuccess) {
            rec->cand = ch.candidate;
            rec->pending = true;
            ++p->pending[ch.candidate];
            ++p->ring_count;
        } else {
            (void)cudaGetLastError();
        }
    }
    ch.exchange = PEPP_X_NONE;
    if (exchanging) {
        const int ex = ((flags & PEPP_Y_REPLICATED) || ex_call == PEPP_X_ALLGATHER) ? PEPP_X_ALLGATHER : PEPP_X_HALO;
        s = ex == PEPP_X_ALLGATHER ? exchange_allgather(p, y, st) : exchange_halo(p, y, st);
        if (!s && ex == PEPP_X_HALO) s = dist_complete(p, y, st, N, &ch.launches);
        if (s) { p->sticky = s; return s; }
        ch.exchange = ex;
        if (ex == PEPP_X_HALO) ch.launches += halo_kernels(p);
    }
    if (scr && (s = scratch_release(p, st))) { p->sticky = s; return s; }
    ++p->ncalls;
    if (used) *used = ch;
    return PEPP_OK;
}

namespace {
constexpr int32_t kDistVariant = 5;   // history uid of a distribution candidate: kDistVariant << 20 | P' << 4 | exchange

int32_t dist_uid(int parts, int ex) { return (kDistVariant << 20) | ((parts & 0xFFFF) << 4) | (ex & 0xF); }

// Time one candidate (P', ex) on this rank: NEXT_INPUT calls on scratch
// vectors until every rank's plans for it finished calibrating their variant
// choice (agreed every 4 calls), then `ms` timed calls (events on the
// stream around the whole call: kernels + exchange). Collective.
pepp_status_t dist_time(pepp_spmv_plan_t* p, int parts, int ex, void* a, void* b, cudaStream_t st, int ms,
                        double* samples) {
    pepp_choice_t f{};
    f.variant = PEPP_V_AUTO;
    f.param = 0;
    f.nparts = parts;
    f.exchange = ex;
    pepp_status_t s;
    for (int it = 0;; it += 4) {
        for (int j = 0; j < 4; ++j) {
            if ((s = pepp_spmv_exec(p, a, b, PEPP_Y_NEXT_INPUT, st, &f, nullptr))) return s;
            std::swap(a, b);
        }
        int64_t busy = dist_busy(p, parts, ex == PEPP_X_P2P ? PEPP_X_HALO : ex) ? 1 : 0;
        if ((s = nccl_allmax(p, st, &busy))) return s;
        if (!busy || it >= 256) break;
    }
    std::vector<cudaEvent_t> ev(2 * ms, nullptr);
    struct Ev { std::vector<cudaEvent_t>& v; ~Ev() { for (auto e : v) if (e) cudaEventDestroy(e); } } guard{ev};
    for (auto& e : ev) PEPP_CUDA_TRY(cudaEventCreate(&e));
    for (int j = 0; j < ms; ++j) {
        PEPP_CUDA_TRY(cudaEventRecord(ev[2 * j], st));
        if ((s = pepp_spmv_exec(p, a, b, PEPP_Y_NEXT_INPUT | PEPP_EXEC_NO_TIMING, st, &f, nullptr))) return s;
        PEPP_CUDA_TRY(cudaEventRecord(ev[2 * j + 1], st));
        std::swap(a, b);
    }
    PEPP_CUDA_TRY(cudaStreamSynchronize(st));
    for (int j = 0; j < ms; ++j) {
        float t = 0.f;
        PEPP_CUDA_TRY(cudaEventElapsedTime(&t, ev[2 * j], ev[2 * j + 1]));
        samples[j] = (double)t * 1000.0;
    }
    return PEPP_OK;
}

// Plan-time choice of (P', exchange) for a partitioned plan (opts.dist_select;
// §8(a) a4; dynamic composition from recorded history, §III P@10254). The
// candidates: P' = nranks first, then every prepared P' < nranks, descending,
// each with halo and allgather (only opts.exchange when it is not AUTO). If
// this rank's loaded history lacks min_samples records of some candidate on
// any rank, every candidate is timed (dist_time) on plan-owned zero vectors
// (SpMV time does not depend on the values) and the samples are max-reduced
// over ranks (a partitioned call lasts as long as its slowest rank) and
// recorded; then the agreed means (this rank's history means, max-reduced)
// give the argmin for NEXT_INPUT calls and, among allgather candidates, for
// REPLICATED calls — identical on every rank (pepp::dist_argmin, the rule of
// pepp_dist_choose).
pepp_status_t dist_probe(pepp_spmv_plan_t* p) {
    PEPP_NVTX("pepp dist probe");
    const int N = p->opts.nranks;
    const double t0 = now_ms();
    std::vector<int> exs;
    if (p->opts.exchange == PEPP_X_HALO || p->opts.exchange == PEPP_X_ALLGATHER) exs = {p->opts.exchange};
    else exs = {PEPP_X_HALO, PEPP_X_ALLGATHER};
    p->dcands.clear();
    for (int ex : exs) p->dcands.push_back({N, ex});
    for (auto it = p->dparts.rbegin(); it != p->dparts.rend(); ++it)
        for (int ex : exs) p->dcands.push_back({it->parts, ex});
    const int nd = (int)p->dcands.size();
    const int ms = std::max(1, p->opts.min_samples);
    p->dist_key = pepp::context_key(p->global_rows, p->ncols, p->global_nnz, 0.0, N,
                                    (p->vt == PEPP_VALUE_F32 ? PEPP_KEY_F32 : 0) |
                                    (p->opts.compress_values ? PEPP_KEY_COMPRESS : 0) | PEPP_KEY_DIST);
    cudaStream_t st = nullptr;
    PEPP_CUDA_TRY(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    struct SG { cudaStream_t s; ~SG() { cudaStreamDestroy(s); } } sg{st};
    pepp_status_t s;
    int64_t need = 0;
    for (const auto& c : p->dcands) {
        const pepp::Welford* w = pepp::history_get(p->hist, p->dist_key, dist_uid(c.parts, c.ex));
        need |= !w || w->count < ms;
    }
    if ((s = nccl_allmax(p, st, &need))) return s;
    if (need) {
        DevTmp<unsigned char> a, b;
        const size_t bytes = (size_t)std::max<int64_t>(1, p->global_rows) * p->esz;
        PEPP_CUDA_TRY(a.alloc(bytes));
        PEPP_CUDA_TRY(b.alloc(bytes));
        PEPP_CUDA_TRY(cudaMemsetAsync(a.p, 0, bytes, st));
        PEPP_CUDA_TRY(cudaMemsetAsync(b.p, 0, bytes, st));
        std::vector<double> samples((size_t)nd * ms, 0.0);
        for (int d = 0; d < nd; ++d)
            if ((s = dist_time(p, p->dcands[d].parts, p->dcands[d].ex, a.p, b.p, st, ms, &samples[(size_t)d * ms]))) return s;
        if ((s = nccl_allmax_f64(p, st, samples))) return s;
        for (int d = 0; d < nd; ++d)
            for (int j = 0; j < ms; ++j)
                pepp::history_add(p->hist, p->dist_key, dist_uid(p->dcands[d].parts, p->dcands[d].ex), samples[(size_t)d * ms + j]);
    }
    std::vector<double> mean(nd, 0.0);
    for (int d = 0; d < nd; ++d) {
        const pepp::Welford* w = pepp::history_get(p->hist, p->dist_key, dist_uid(p->dcands[d].parts, p->dcands[d].ex));
        mean[d] = w ? w->mean : 0.0;
    }
    if ((s = nccl_allmax_f64(p, st, mean))) return s;
    p->dist_agreed = mean;
    std::vector<uint8_t> ag(nd);
    for (int d = 0; d < nd; ++d) ag[d] = p->dcands[d].ex == PEPP_X_ALLGATHER;
    p->dist_next = pepp::dist_argmin(nd, mean.data(), nullptr);
    p->dist_repl = pepp::dist_argmin(nd, mean.data(), ag.data());
    if (p->dist_next < 0) p->dist_next = 0;
    pepp_plan_info_t& I = p->info;
    I.dist_candidates = nd;
    I.dist_nparts = p->dcands[p->dist_next].parts;
    I.dist_exchange = p->dcands[p->dist_next].ex;
    I.dist_repl_nparts = p->dist_repl >= 0 ? p->dcands[p->dist_repl].parts : N;
    I.dist_probe_ms = now_ms() - t0;
    return PEPP_OK;
}

// The fused push as a distribution candidate (P' = nranks, PEPP_X_P2P), timed
// on the just-registered buffers like dist_probe's candidates and compared
// with the agreed best (1 % tie rule: the NCCL candidates come first).
pepp_status_t p2p_probe(pepp_spmv_plan_t* p) {
    PEPP_NVTX("pepp p2p probe");
    const int N = p->opts.nranks, ms = std::max(1, p->opts.min_samples);
    cudaStream_t st = nullptr;
    PEPP_CUDA_TRY(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    struct SG { cudaStream_t s; ~SG() { cudaStreamDestroy(s); } } sg{st};
    pepp_status_t s;
    const int32_t uid = dist_uid(N, PEPP_X_P2P);
    const pepp::Welford* w = pepp::history_get(p->hist, p->dist_key, uid);
    int64_t need = !w || w->count < ms;
    if ((s = nccl_allmax(p, st, &need))) return s;
    if (need && p->p2p_nbuf < 2) return PEPP_OK;   // one buffer: no ping-pong to time it with; the push is used
    if (need) {
        std::vector<double> samples(ms, 0.0);
        const bool keep = p->p2p_use;
        p->p2p_use = true;
        s = dist_time(p, N, PEPP_X_P2P, p->p2p_buf[0], p->p2p_buf[1 % p->p2p_nbuf], st, ms, samples.data());
        p->p2p_use = keep;
        if (s) return s;
        if ((s = nccl_allmax_f64(p, st, samples))) return s;
        for (double v : samples) pepp::history_add(p->hist, p->dist_key, uid, v);
    }
    std::vector<double> m(1, pepp::history_get(p->hist, p->dist_key, uid)->mean);
    if ((s = nccl_allmax_f64(p, st, m))) return s;
    p->p2p_agreed = m[0];
    const double best = p->dist_next >= 0 ? p->dist_agreed[p->dist_next] : 0.0;
    p->p2p_use = !(best > 0.0) || m[0] < best * 0.99;
    if (p->p2p_use) { p->info.dist_nparts = N; p->info.dist_exchange = PEPP_X_P2P; }
    return PEPP_OK;
}
}  // namespace

struct pepp_spmv_graph_s {
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t exec = nullptr;
    int device = 0;
};

extern "C" PEPP_API pepp_status_t pepp_spmv_graph_create(pepp_spmv_plan_t* p, const void* x, void* y, void* work,
                                                        int32_t iterations, int32_t mode, int flags, void* stream,
                                                        pepp_spmv_graph_t** out) {
    if (!out) return PEPP_E_INVALID;
    *out = nullptr;
    if (!p || iterations < 1 || (mode != 0 && mode != 1) || (mode == 1 && iterations > 1 && !work)) return PEPP_E_INVALID;
    if (mode == 1 && p->ncols != p->global_rows) return PEPP_E_INVALID;
    if (p->sticky) return p->sticky;
    DeviceScope dscope(p->device);
    if (!dscope.ok) return PEPP_E_CUDA;
    // choose once, outside the capture: the best measured candidate so far,
    // else the heuristic (frozen: a calibration pick would be baked into
    // every replay untimed)
    pepp_choice_t ch{};
    pepp_status_t s = select_choice(p, &ch, /*frozen=*/true);
    if (s) return s;
    cudaStream_t st = (cudaStream_t)stream;
    cudaStream_t cap = nullptr;
    if (cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking) != cudaSuccess) { (void)cudaGetLastError(); return PEPP_E_CUDA; }
    pepp_spmv_graph_t* g = new (std::nothrow) pepp_spmv_graph_t();
    if (!g) { cudaStreamDestroy(cap); return PEPP_E_NOMEM; }
    g->device = p->device;
    bool ok = cudaStreamBeginCapture(cap, cudaStreamCaptureModeRelaxed) == cudaSuccess;
    const void* in = x;
    void* outb = y;
    for (int32_t it = 0; ok && it < iterations; ++it) {
        s = pepp_spmv_exec(p, in, outb, flags | PEPP_EXEC_NO_TIMING, cap, &ch, nullptr);
        if (s) ok = false;
        if (mode == 1) {
            in = outb;
            outb = (outb == y) ? work : y;
        }
    }
    cudaGraph_t graph = nullptr;
    const bool ended = cudaStreamEndCapture(cap, &graph) == cudaSuccess;
    cudaStreamDestroy(cap);
    if (!ok || !ended || !graph) {
        (void)cudaGetLastError();
        if (graph) cudaGraphDestroy(graph);
        delete g;
        return s ? s : PEPP_E_CUDA;
    }
    g->graph = graph;
    if (cudaGraphInstantiate(&g->exec, graph, 0) != cudaSuccess) {
        (void)cudaGetLastError();
        cudaGraphDestroy(graph);
        delete g;
        return PEPP_E_CUDA;
    }
    if (cudaGraphUpload(g->exec, st) != cudaSuccess) (void)cudaGetLastError();   // pre-stage on the caller's stream
    *out = g;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_graph_launch(pepp_spmv_graph_t* g, void* stream) {
    if (!g) return PEPP_E_INVALID;
    DeviceScope dscope(g->device);
    if (!dscope.ok || cudaGraphLaunch(g->exec, (cudaStream_t)stream) != cudaSuccess) {
        (void)cudaGetLastError();
        return PEPP_E_CUDA;
    }
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_graph_destroy(pepp_spmv_graph_t* g) {
    if (!g) return PEPP_OK;
    DeviceScope dscope(g->device);
    if (g->exec) cudaGraphExecDestroy(g->exec);
    if (g->graph) cudaGraphDestroy(g->graph);
    delete g;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_exec_vec(pepp_spmv_plan_t* p, pepp_vector_t* x, pepp_vector_t* y, int flags,
                                                    void* stream, const pepp_choice_t* force, pepp_choice_t* used) {
    if (!p || !x || !y || x == y) return PEPP_E_INVALID;
    if (p->vt != PEPP_VALUE_F64) return PEPP_E_UNSUPPORTED;   // containers hold fp64
    if (pepp::vector_simulated(x) || pepp::vector_simulated(y)) return PEPP_E_INVALID;
    if (pepp::vector_length(x) != p->ncols || pepp::vector_length(y) != p->global_rows) return PEPP_E_INVALID;
    double *dx = nullptr, *dy = nullptr;
    pepp_status_t s = pepp_vector_acquire_device(x, PEPP_ACCESS_READ, stream, &dx);
    if (s) return s;
    // y is written (A4). Every global row is written only when the call ends
    // with an allgather (PEPP_Y_REPLICATED, or NEXT_INPUT on an allgather
    // plan) or the plan is unpartitioned; a partitioned LOCAL or halo call
    // writes this block's rows (+ ghosts) and leaves the rest as they were,
    // so y is READWRITE there: its device copy must hold the current values
    // of the rows the call does not write before the whole buffer becomes the
    // valid copy
    const bool all_rows = p->opts.nranks == 1 || (flags & PEPP_Y_REPLICATED) ||
                          ((flags & PEPP_Y_NEXT_INPUT) && p->exchange == PEPP_X_ALLGATHER);
    s = pepp_vector_acquire_device(y, all_rows ? PEPP_ACCESS_WRITE : PEPP_ACCESS_READWRITE, stream, &dy);
    if (s) return s;
    s = pepp_spmv_exec(p, dx, dy, flags, stream, force, used);
    const pepp_status_t s1 = pepp_vector_release_device(x, stream);
    const pepp_status_t s2 = pepp_vector_release_device(y, stream);
    return s ? s : (s1 ? s1 : s2);
}

extern "C" PEPP_API pepp_status_t pepp_spmv_exchange(pepp_spmv_plan_t* p, void* y, int flags, void* stream) {
    PEPP_NVTX("pepp_spmv_exchange");
    if (!p) return PEPP_E_INVALID;
    if (p->sticky) return p->sticky;
    if (p->opts.nranks == 1 || !(flags & (PEPP_Y_NEXT_INPUT | PEPP_Y_REPLICATED))) return PEPP_OK;
    if (!y) return PEPP_E_INVALID;
    DeviceScope dscope(p->device);
    if (!dscope.ok) return PEPP_E_CUDA;
    cudaStream_t st = (cudaStream_t)stream;
    const bool ag = (flags & PEPP_Y_REPLICATED) || p->exchange == PEPP_X_ALLGATHER;
    pepp_status_t s = ag ? exchange_allgather(p, y, st) : exchange_halo(p, y, st);
    if (!s && !ag) s = dist_complete(p, y, st, p->opts.nranks, nullptr);
    if (s) p->sticky = s;
    return s;
}

namespace {
// `iterations` calls x_{k+1} = A·x_k starting from device buffer a (b is the
// other iteration buffer); *out gets the buffer holding the final y
pepp_status_t host_iterations(pepp_spmv_plan_t* p, void* a, void* b, int32_t iterations, int flags, cudaStream_t st,
                              void** out) {
    void *xin = a, *yout = b;
    for (int32_t it = 0; it < iterations; ++it) {
        const bool last = it == iterations - 1;
        const int f = last ? flags : (flags & PEPP_EXEC_NO_TIMING) | PEPP_Y_NEXT_INPUT;
        pepp_status_t s = pepp_spmv_exec(p, xin, yout, f, st, nullptr, nullptr);
        if (s) return s;
        if (!last) std::swap(xin, yout);
    }
    *out = yout;
    return PEPP_OK;
}

// rows copied back: all global rows with PEPP_Y_REPLICATED, else this rank's rows
void host_rows(const pepp_spmv_plan_t* p, int flags, int64_t* lo, int64_t* cnt) {
    *lo = p->row_offset;
    *cnt = p->nrows;
    if (p->opts.nranks > 1 && (flags & PEPP_Y_REPLICATED)) { *lo = 0; *cnt = p->global_rows; }
}
}  // namespace

extern "C" PEPP_API pepp_status_t pepp_spmv_exec_host(pepp_spmv_plan_t* p, const void* x_host, void* y_host,
                                                     int32_t iterations, int flags, void* stream) {
    PEPP_NVTX("pepp_spmv_exec_host");
    if (!p || !x_host || !y_host || iterations < 1) return PEPP_E_INVALID;
    if (p->sticky) return p->sticky;
    if (iterations > 1 && p->ncols != p->global_rows) return PEPP_E_INVALID;
    cudaStream_t st = (cudaStream_t)stream;
    DeviceScope dscope(p->device);
    if (!dscope.ok) return PEPP_E_CUDA;
    const int64_t nx = std::max<int64_t>(p->ncols, p->global_rows);
    if (!p->d_hx) {
        pepp_status_t s;
        if ((s = dalloc_bytes(p, &p->d_hx, nx * (int64_t)p->esz))) return s;
        if ((s = dalloc_bytes(p, &p->d_hy, nx * (int64_t)p->esz))) return s;
    }
    auto enqueue = [&]() -> pepp_status_t {
        PEPP_CUDA_TRY(cudaMemcpyAsync(p->d_hx, x_host, p->esz * p->ncols, cudaMemcpyHostToDevice, st));
        void* yout = nullptr;
        pepp_status_t s = host_iterations(p, p->d_hx, p->d_hy, iterations, flags, st, &yout);
        if (s) return s;
        int64_t lo, cnt;
        host_rows(p, flags, &lo, &cnt);
        if (cnt > 0)
            PEPP_CUDA_TRY(cudaMemcpyAsync((char*)y_host + lo * (int64_t)p->esz, (const char*)yout + lo * (int64_t)p->esz,
                                          p->esz * cnt, cudaMemcpyDeviceToHost, st));
        return PEPP_OK;
    };
    const pepp_status_t s = enqueue();
    // also on failure: nothing queued may still touch the caller's host buffers
    if (cudaStreamSynchronize(st) != cudaSuccess) { (void)cudaGetLastError(); p->sticky = PEPP_E_CUDA; return PEPP_E_CUDA; }
    return s;
}

// Software pipeline over independent right-hand sides: item k's host->device
// copy (stream cs_in), its iterations (the caller's stream) and its
// device->host copy (stream cs_out) use slot k % 2, so item k+1's input copy
// and item k-1's output copy run on the copy engines while item k computes.
// A slot is refilled only after its previous output copy finished (ev_free).
extern "C" PEPP_API pepp_status_t pepp_spmv_exec_host_batch(pepp_spmv_plan_t* p, int32_t nbatch,
                                                           const void* const* x_hosts, void* const* y_hosts,
                                                           int32_t iterations, int flags, void* stream) {
    PEPP_NVTX("pepp_spmv_exec_host_batch");
    if (!p || nbatch < 0 || (nbatch > 0 && (!x_hosts || !y_hosts)) || iterations < 1) return PEPP_E_INVALID;
    for (int32_t k = 0; k < nbatch; ++k) if (!x_hosts[k] || !y_hosts[k]) return PEPP_E_INVALID;
    if (p->sticky) return p->sticky;
    if (iterations > 1 && p->ncols != p->global_rows) return PEPP_E_INVALID;
    if (nbatch == 0) return PEPP_OK;
    if (nbatch == 1) return pepp_spmv_exec_host(p, x_hosts[0], y_hosts[0], iterations, flags, stream);
    cudaStream_t st = (cudaStream_t)stream;
    DeviceScope dscope(p->device);
    if (!dscope.ok) return PEPP_E_CUDA;
    const int64_t nx = std::max<int64_t>(p->ncols, p->global_rows);
    // first use: slots, copy streams, events (each created once; a failed
    // attempt leaves what it made for the next one, nothing leaks)
    for (void*& b : p->d_hb)
        if (!b) {
            pepp_status_t s = dalloc_bytes(p, &b, nx * (int64_t)p->esz);
            if (s) return s;
        }
    for (cudaStream_t* q : {&p->cs_in, &p->cs_out})
        if (!*q) PEPP_CUDA_TRY(cudaStreamCreateWithFlags(q, cudaStreamNonBlocking));
    for (cudaEvent_t* e : {&p->ev_start, &p->ev_end, &p->ev_in[0], &p->ev_in[1], &p->ev_out[0], &p->ev_out[1],
                           &p->ev_free[0], &p->ev_free[1]})
        if (!*e) PEPP_CUDA_TRY(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
    int64_t lo, cnt;
    host_rows(p, flags, &lo, &cnt);
    auto enqueue = [&]() -> pepp_status_t {
        // the copies start after everything the caller queued on its stream
        PEPP_CUDA_TRY(cudaEventRecord(p->ev_start, st));
        PEPP_CUDA_TRY(cudaStreamWaitEvent(p->cs_in, p->ev_start, 0));
        PEPP_CUDA_TRY(cudaStreamWaitEvent(p->cs_out, p->ev_start, 0));
        for (int32_t k = 0; k < nbatch; ++k) {
            const int b = k & 1;
            void *xa = p->d_hb[2 * b], *xb = p->d_hb[2 * b + 1];
            if (k >= 2) PEPP_CUDA_TRY(cudaStreamWaitEvent(p->cs_in, p->ev_free[b], 0));
            PEPP_CUDA_TRY(cudaMemcpyAsync(xa, x_hosts[k], p->esz * p->ncols, cudaMemcpyHostToDevice, p->cs_in));
            PEPP_CUDA_TRY(cudaEventRecord(p->ev_in[b], p->cs_in));
            PEPP_CUDA_TRY(cudaStreamWaitEvent(st, p->ev_in[b], 0));
            void* yout = nullptr;
            pepp_status_t s = host_iterations(p, xa, xb, iterations, flags, st, &yout);
            if (s) return s;
            PEPP_CUDA_TRY(cudaEventRecord(p->ev_out[b], st));
            PEPP_CUDA_TRY(cudaStreamWaitEvent(p->cs_out, p->ev_out[b], 0));
            if (cnt > 0)
                PEPP_CUDA_TRY(cudaMemcpyAsync((char*)y_hosts[k] + lo * (int64_t)p->esz,
                                              (const char*)yout + lo * (int64_t)p->esz, p->esz * cnt,
                                              cudaMemcpyDeviceToHost, p->cs_out));
            PEPP_CUDA_TRY(cudaEventRecord(p->ev_free[b], p->cs_out));
        }
        PEPP_CUDA_TRY(cudaEventRecord(p->ev_end, p->cs_out));
        PEPP_CUDA_TRY(cudaStreamWaitEvent(st, p->ev_end, 0));
        return PEPP_OK;
    };
    const pepp_status_t s = enqueue();
    // on success the caller's stream has joined the copy streams; on failure
    // drain all three so no copy still touches the caller's host buffers
    bool ok = cudaStreamSynchronize(st) == cudaSuccess;
    if (s) {
        ok &= cudaStreamSynchronize(p->cs_in) == cudaSuccess;
        ok &= cudaStreamSynchronize(p->cs_out) == cudaSuccess;
    }
    if (!ok) { (void)cudaGetLastError(); p->sticky = PEPP_E_CUDA; return PEPP_E_CUDA; }
    return s;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_destroy(pepp_spmv_plan_t* p) {
    if (!p) return PEPP_OK;
    DeviceScope dscope(p->device);
    harvest(p, true);
    cudaDeviceSynchronize();
    (void)cudaGetLastError();
    pepp_status_t s = PEPP_OK;
    if (p->p2p_nbuf && p->nccl && p->comm) {   // peers may still write into this rank's buffers
        cudaStream_t st = nullptr;
        if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) == cudaSuccess) {
            s = nccl_barrier(p, st);
            cudaStreamDestroy(st);
        }
        (void)cudaGetLastError();
    }
    if (!p->history_path.empty() && p->hist) s = pepp_history_save(p->hist, p->history_path.c_str());
    free_plan(p);
    return s;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_p2p_buffers(pepp_spmv_plan_t* p, int32_t nbuf, void** bufs) {
    PEPP_NVTX("pepp_spmv_p2p_buffers");
    if (!p || !bufs || nbuf < 1 || nbuf > kP2PMaxBuf) return PEPP_E_INVALID;
    if (p->sticky) return p->sticky;
    if (p->p2p_nbuf) return PEPP_E_STATE;
    if (p->opts.nranks < 2) return PEPP_E_UNSUPPORTED;
    DeviceScope dscope(p->device);
    if (!dscope.ok) { pepp::set_last_error("cannot select the plan's device", "DeviceScope", __LINE__); return PEPP_E_CUDA; }
    cudaStream_t st = nullptr;
    PEPP_CUDA_TRY(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    // agreement first (collective on every path): a rank that cannot take
    // part — no halo exchange, or rows it sends outside a head / tail split —
    // makes every rank return PEPP_E_UNSUPPORTED before any rank enters the
    // registration collectives
    int64_t cant = (p->exchange != PEPP_X_HALO || !p2p_capable(p)) ? 1 : 0;
    pepp_status_t s = nccl_allmax(p, st, &cant);
    if (!s && cant) s = PEPP_E_UNSUPPORTED;
    else if (!s) s = p2p_register(p, nbuf, st);
    cudaStreamDestroy(st);
    if (s == PEPP_E_UNSUPPORTED) return s;   // nothing changed: the plan stays usable (NCCL halo)
    if (s && s != PEPP_E_NCCL) {
        // every rank saw the failure through the agreement max-reduce: undo,
        // and the plan keeps working with the NCCL halo (not sticky)
        p2p_reset(p);
        return s;
    }
    if (s) { p->sticky = s; return s; }
    // the fused push is a timed distribution candidate too (collective)
    if (!p->dcands.empty() && (s = p2p_probe(p))) { p->sticky = s; return s; }
    for (int b = 0; b < nbuf; ++b) bufs[b] = p->p2p_buf[b];
    p->info.p2p_buffers = nbuf;
    p->info.device_bytes = p->dev_bytes;
    for (auto* q : p->sub) if (q) p->info.device_bytes += q->dev_bytes;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_plan_info(const pepp_spmv_plan_t* p, pepp_plan_info_t* out) {
    if (!p || !out) return PEPP_E_INVALID;
    *out = p->info;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_candidates(const pepp_spmv_plan_t* p, pepp_choice_t* out, int32_t cap,
                                                      int32_t* n) {
    if (!p || !n) return PEPP_E_INVALID;
    *n = (int32_t)p->cands.size();
    for (int32_t i = 0; out && i < cap && i < *n; ++i) {
        fill_choice(p, i, 0, 0.0, &out[i]);
        const pepp::Welford* w = pepp::history_get(p->hist, p->key, p->uids[i]);
        out[i].predicted_us = w ? w->mean : (p->prior[i] > 0 ? p->prior[i] : 0.0);
    }
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_dist_stats(const pepp_spmv_plan_t* p, int32_t cap, int32_t* nparts,
                                                      int32_t* exchange, double* agreed_us, int32_t* n) {
    if (!p || !n || cap < 0) return PEPP_E_INVALID;
    const int32_t nd = (int32_t)p->dcands.size(), tot = nd + (nd && p->p2p_nbuf ? 1 : 0);
    *n = tot;
    for (int32_t i = 0; i < tot && i < cap; ++i) {
        const bool pp = i == nd;
        if (nparts) nparts[i] = pp ? p->opts.nranks : p->dcands[i].parts;
        if (exchange) exchange[i] = pp ? PEPP_X_P2P : p->dcands[i].ex;
        if (agreed_us) agreed_us[i] = pp ? p->p2p_agreed : p->dist_agreed[i];
    }
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_flush_history(pepp_spmv_plan_t* p) {
    if (!p) return PEPP_E_INVALID;
    DeviceScope dscope(p->device);
    harvest(p, true);
    for (auto* q : p->sub) if (q) harvest(q, true);
    for (auto& dp : p->dparts) if (dp.plan) harvest(dp.plan, true);
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_spmv_history_stats(const pepp_spmv_plan_t* p, int32_t cand, int64_t* count,
                                                         double* mean_us, double* m2) {
    if (!p || cand < 0 || cand >= (int32_t)p->cands.size()) return PEPP_E_INVALID;
    return pepp_history_stats(p->hist, p->key, p->uids[cand], count, mean_us, m2);
}
