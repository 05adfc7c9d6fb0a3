/*
 * pepp_spmv.h — C-ABI of the B200-native SpMV hot path (libpepp_spmv.so).
 *
 * The operation is the PEPPHER composition example component
 *
 *     void spmv(float* values, int nnz, int nrows, int ncols, int first,
 *               size_t* colidxs, size_t* rowPtr, float* x, float* y);
 *
 * (Dastgeer, Li, Kessler, MuCoCoS 2012, §V-A; PAPER.md P@32944 + P@31037 —
 * the signature is split by the PDF extraction, garble G1 of SURVEY.md §0):
 *
 *     y[i] = Σ_{k = rowPtr[i]-first}^{rowPtr[i+1]-first-1} values[k] · x[colidxs[k]]
 *
 * re-designed as plan / select / exec / destroy:
 *   - pepp_spmv_plan    ~ PEPPHER_INITIALIZE + smart-container registration
 *                          ("register once", §IV-H P@28291–29611): validates,
 *                          extracts the context instance (§III P@9781),
 *                          copies the operand into device memory it owns and
 *                          prepares every implementation variant (§II P@4772).
 *   - pepp_spmv_select  ~ the runtime's performance-aware variant choice from
 *                          recorded history (dynamic composition §III
 *                          P@10254–10489; useHistoryModels P@28038, P@29611).
 *   - pepp_spmv_exec    ~ the generated entry-wrapper (§IV-C P@16839): one call,
 *                          asynchronous (P@17990), partitioned over ranks whose
 *                          outputs concatenate (§IV-F P@27330–28000).
 *   - pepp_spmv_destroy ~ PEPPHER_SHUTDOWN (P@33881).
 *
 * Precision and index widths (readings A2, A3): values, x, y and all
 * sums are fp64 (PEPP_VALUE_F64, the default) or — the paper's own `float`
 * signature (P@32944), SURVEY §8(f) f3 — fp32 throughout (PEPP_VALUE_F32:
 * fp32 values, x, y, products and sums); the value type is a property of the
 * plan and every value pointer below (x, y, work, host buffers) points to
 * elements of that type. Column indices int32; row pointers int64 at the ABI
 * (the paper's size_t) — narrowed to int32 on the device (nnz < 2^31
 * required; larger blocks return PEPP_E_UNSUPPORTED).
 *
 * Access modes follow the paper's interface descriptor (read / write /
 * readwrite, §II P@4233) and the const / non-const inference of the utility
 * mode (§IV-I P@31894): every `const T*` argument is READ, `double* y` is
 * WRITE (not read; y = A·x, not y += A·x — reading A4).
 *
 * Errors: every entry point returns pepp_status_t; no abort, no exception and
 * no exit crosses the ABI. A CUDA error inside a plan is sticky for that plan
 * (PEPP_E_CUDA on every later call), like a CUDA context error.
 * Threading: a plan is not thread-safe; distinct plans are independent.
 * Streams: one plan may be called on several streams with no synchronisation
 * in between. Candidates that use the plan's device scratch (merge-path and
 * CSR-stream carries, hybrid-SELL partial sums, halo buffers) are ordered
 * across streams by the plan (each such call waits for the previous one on
 * another stream); scratch-free calls overlap (inter-call parallelism,
 * P@21908–27091). Inside a CUDA graph capture that ordering is the graph's.
 * There is NO CPU fallback: a machine without a CUDA device gets PEPP_E_CUDA
 * from pepp_spmv_plan. The host-only utilities at the end of this header
 * (partition, halo lists, history/selector) run without a GPU.
 */
#ifndef PEPP_SPMV_H
#define PEPP_SPMV_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PEPP_ABI_VERSION 10

typedef enum {
    PEPP_OK = 0,
    PEPP_E_INVALID = -1,      /* bad argument or malformed CSR              */
    PEPP_E_CUDA = -2,         /* CUDA runtime error (sticky per plan)       */
    PEPP_E_NCCL = -3,         /* NCCL missing or failed                     */
    PEPP_E_NOMEM = -4,        /* host or device allocation failed          */
    PEPP_E_UNSUPPORTED = -5,  /* valid but not supported (e.g. nnz >= 2^31) */
    PEPP_E_STATE = -6         /* call not valid in the object's state       */
} pepp_status_t;

/* Implementation variants (§II P@4772: "several implementations of one
   interface"; the paper's CUSP variant P@33595 is replaced by four
   hand-written sm_100a kernels). */
typedef enum {
    PEPP_V_AUTO = -1,
    PEPP_V_CSR_VECTOR = 0,    /* TPR lanes per row, 128-bit val/col loads, shfl_xor reduction; param = TPR */
    PEPP_V_MERGE_PATH = 1,    /* merge-path over (row ends, nnz), smem-staged, deterministic carry fix-up */
    PEPP_V_SELL = 2,          /* SELL-C-σ, C = 32, column-major chunks; param = σ */
    PEPP_V_CSR_STREAM = 3,    /* CSR-stream fed by a TMA (cp.async.bulk) shared-memory pipeline; param = nnz per item */
    PEPP_V_PANEL = 4,         /* column panels for x far beyond L2 (random columns): the matrix stored panel-major,
                                 one launch per panel of 2^param columns, (row, panel) pairs summed in order
                                 (deterministic, no atomics); a candidate only when ncols x value size > 96 MB
                                 and the mean row span exceeds half a panel; param = log2 panel width */
    PEPP_V_COUNT = 5
} pepp_variant_t;

/* Exchange that makes y usable as the next x when the call is partitioned */
typedef enum {
    PEPP_X_AUTO = -1,
    PEPP_X_NONE = 0,          /* single rank                                          */
    PEPP_X_ALLGATHER = 1,     /* allgatherv of y slices: every rank gets all of y     */
    PEPP_X_HALO = 2,          /* ghost (halo) exchange: only entries peers' rows read */
    PEPP_X_P2P = 3            /* halo written by the boundary-row kernel itself straight into the
                                 peers' registered buffers over peer memory (CUDA IPC mappings:
                                 NVLink / NVSwitch stores), signalled with flags in peer memory —
                                 compute and exchange in one kernel, no NCCL on the data path.
                                 Used (never requested) by PEPP_Y_NEXT_INPUT calls whose y is one
                                 of the plan's pepp_spmv_p2p_buffers; reported in pepp_choice_t */
} pepp_exchange_t;

/* value types (pepp_csr_t.value_type) */
#define PEPP_VALUE_F64 0
#define PEPP_VALUE_F32 1

/* exec flags: which part of y is valid on return (once the stream completes) */
#define PEPP_Y_LOCAL       0x0  /* own rows only: y[row_offset, row_offset+nrows)              */
#define PEPP_Y_NEXT_INPUT  0x1  /* own rows + every entry this plan's next call reads as x     */
#define PEPP_Y_REPLICATED  0x2  /* all global rows (allgatherv)                                */
#define PEPP_EXEC_NO_TIMING 0x10 /* do not record event timing for this call (e.g. graph capture) */

/* CSR operand (the paper's tuple, G1). Row i of this block holds entries
   [row_ptr[i] - first, row_ptr[i+1] - first) of col_idx / values (reading
   A1: `first` is the row-pointer base, so a rank can pass a slice of a
   global rowPtr unchanged; column indices are 0-based and global).
   Invariants checked by pepp_spmv_plan: row_ptr[0] == first,
   row_ptr[nrows] - first == nnz, row_ptr non-decreasing, 0 <= col < ncols.
   Duplicate or unsorted columns within a row are allowed and summed (A8).
   All three arrays are READ; host memory if on_device == 0, else device
   memory on the plan's device. The plan copies what it needs: the caller may
   free them as soon as pepp_spmv_plan returns. */
typedef struct {
    int64_t nrows;            /* rows in this block                          */
    int64_t ncols;            /* columns = length of x (global)              */
    int64_t nnz;              /* entries in this block                       */
    int64_t first;            /* row_ptr base (paper's `first`)              */
    const int64_t* row_ptr;   /* [nrows + 1]                                 */
    const int32_t* col_idx;   /* [nnz]                                       */
    const void* values;       /* [nnz] of value_type                         */
    int32_t on_device;        /* 0 = host pointers, 1 = device pointers      */
    int32_t value_type;       /* PEPP_VALUE_F64 (0, default) or PEPP_VALUE_F32 */
} pepp_csr_t;

struct pepp_plan_info_s;   /* = pepp_plan_info_t, below */

/* Performance prediction function (the component descriptor's "reference to a
   (usually, programmer provided) performance prediction function that is
   called with a given context descriptor data structure", §II P@6887–7157).
   Called at plan time, once per candidate, with the plan's context instance
   (`context`: sizes, row statistics, key; the candidate list is not final
   yet) and the candidate's variant and tunable; returns the predicted time of
   one call in µs, or <= 0 for "no prediction". Must not call back into the
   plan. `user` is opts.predict_user. */
typedef double (*pepp_predict_fn)(const struct pepp_plan_info_s* context, int32_t variant, int32_t param,
                                  void* user);

/* Plan options. Use pepp_spmv_opts_default() then override. */
typedef struct {
    uint32_t variant_mask;    /* bit v set = variant v allowed; 0 = all (the paper's disableImpls, P@16687) */
    int32_t use_history;      /* 1 = history-based dynamic selection (default; useHistoryModels P@28038);
                                 0 = fixed heuristic from the context instance */
    int32_t validate;         /* 1 = full O(nnz) check of the CSR invariants (default) */
    int32_t sell_sigma;       /* SELL sorting window σ (rows); 0 = chosen from the padding ratio */
    int32_t device;           /* CUDA device ordinal; -1 = the caller's current device */
    int32_t min_samples;      /* timed calls per candidate before exploiting (default 3) */
    int32_t sample_period;    /* after calibration, time every N-th call (default 8; 0 = never) */
    /* partitioning (§IV-F intra-component parallelism, P@27330–28000) */
    int32_t nranks;           /* ranks the global matrix is split over (1 = unpartitioned) */
    int32_t rank;             /* this process's rank */
    const int64_t* row_bounds;/* [nranks + 1] global row boundaries (x is split the same way; square A);
                                 NULL when nranks == 1. This block is rows [row_bounds[rank], row_bounds[rank+1]) */
    void* nccl_comm;          /* borrowed ncclComm_t, or NULL */
    const void* nccl_unique_id; /* 128-byte ncclUniqueId (same on every rank) when nccl_comm is NULL and nranks > 1 */
    int32_t exchange;         /* pepp_exchange_t; AUTO = halo when ghosts are < 1/4 of ncols, else allgather */
    const char* history_path; /* if set: history loaded at plan, saved at destroy (NEXT-f2 persistence) */
    int32_t prune;            /* 1 (default) = multi-stage composition (P@10489): statically narrow the
                                 candidates from the context instance before the runtime choice —
                                 vector-CSR only if max_row <= max(4096, 256*mean); SELL, merge-path
                                 and CSR-stream always (SELL moves rows longer than
                                 info.sell_cap to its segmented long-row kernel).
                                 0 = every variant is a candidate (variant_mask still applies). */
    int32_t overlap;          /* partitioned halo plans (nranks > 1): 1 (default) = when the rows this
                                 rank sends lie in a short head and tail of its block (stencils, banded
                                 matrices), a PEPP_Y_NEXT_INPUT call computes head and tail first, then
                                 runs the halo exchange on a plan-owned side stream while the interior
                                 rows compute, and joins before returning (the paper's overlap of
                                 communication with computation in partitioned execution, §IV-F
                                 P@27330–28000). Costs a second device copy of the block (head,
                                 interior and tail sub-plans). 0 = kernel, then exchange, in order. */
    pepp_predict_fn predict;  /* optional (NULL = none). Its predictions stand in where no recorded
                                 history exists: with use_history = 1 they order the calibration
                                 (predicted best first) and rule out candidates predicted > 4x the
                                 best prediction, exactly like a cold-start prior from a recorded
                                 context (which takes precedence when both exist); with
                                 use_history = 0 every call dispatches to the argmin of the
                                 predictions (static composition through the prediction function,
                                 P@10069) instead of the built-in heuristic. */
    void* predict_user;       /* passed to predict; borrowed, used only during pepp_spmv_plan */
    int32_t compress_values;  /* 1 (default) = value compression in the SELL layout: a stencil chunk
                                 (32 rows sharing their column offsets) whose every slot holds one
                                 bitwise-identical value for all 32 rows becomes an id into a small
                                 per-plan pattern table (<= 32 patterns of <= 8 slots, passed to the
                                 kernel by value): the chunk then reads only x and writes y
                                 (constant-coefficient stencils). Lossless: the same products and
                                 sums in the same order (bit-identical y); only the bytes read
                                 change. 0 = every stored slot's value is streamed. */
    int32_t dist_select;      /* nranks > 1, use_history = 1: 1 (default) = the partition count P and the
                                 exchange are timed choices too (§8(a) a4; the runtime picks "which
                                 implementation/device to use by considering previous historical
                                 execution information as well as ... load balance, data locality and
                                 potential data-transfer cost", §V-D P@38827). Candidates: P' in the
                                 powers of two dividing nranks (the call runs on ranks 0..P'-1, each on
                                 the union of nranks/P' consecutive row blocks, shipped to it over NCCL
                                 at plan time) x exchange in {halo, allgather} (only opts.exchange when
                                 it is not AUTO), plus the fused peer-memory push once
                                 pepp_spmv_p2p_buffers registers buffers. pepp_spmv_plan (and
                                 pepp_spmv_p2p_buffers) time each candidate with plan-owned scratch
                                 vectors — its kernels first calibrated, then min_samples timed
                                 calls — and all ranks agree on the max-over-ranks means (one NCCL
                                 max-reduce): every later PEPP_Y_NEXT_INPUT call runs the argmin
                                 (PEPP_Y_REPLICATED: the argmin among allgather candidates;
                                 PEPP_Y_LOCAL: always P' = nranks). A loaded history_path with
                                 min_samples records of every candidate on every rank skips the
                                 timing. 0 = P' = nranks, exchange by the plan's footprint rule. */
} pepp_spmv_opts_t;

/* Selection result. `candidate` indexes pepp_spmv_candidates(). The plan's
   history records each candidate under the stable id (variant << 20 | param),
   so a persisted history (history_path) means the same across plans. */
typedef struct {
    int32_t variant;          /* pepp_variant_t */
    int32_t param;            /* TPR (CSR_VECTOR), σ (SELL), items per thread (MERGE_PATH), nnz per item (CSR_STREAM) */
    int32_t nparts;           /* ranks the call runs on */
    int32_t exchange;         /* pepp_exchange_t used when flags ask for it */
    int32_t calibrating;      /* 1 = chosen to gather history, not the predicted best */
    int32_t candidate;        /* index in the plan's candidate list */
    double predicted_us;      /* history mean of this candidate (0 if unknown) */
    int32_t launches;         /* exec only: kernels of this library the call launched (SpMV kernels,
                                 fix-ups, halo pack/unpack or the fused push; NCCL's own not counted) */
    int32_t reserved;
    int64_t layout_bytes;     /* bytes this candidate's kernels move from / to HBM per call with the plan's
                                 layout as stored: matrix arrays as the variant streams them (values,
                                 index stream or per-chunk stencil offsets, descriptors, lists, row
                                 pointers), x read once (ncols) and y written once (nrows) — the
                                 physical roofline numerator. SURVEY §8(d)'s algorithmic bytes
                                 (nnz*12 + row_ptr + x + y) are pepp_plan_info_t.algorithmic_bytes:
                                 a compressed layout streams fewer bytes than that for the same work. */
} pepp_choice_t;

/* Context instance (§III P@9781: "a tuple of concrete values for context
   properties that might influence callee selection") + plan facts. */
typedef struct pepp_plan_info_s {
    int64_t nrows, ncols, nnz;
    double mean_row;          /* nnz / nrows */
    double cv_row;            /* coefficient of variation of row lengths */
    int64_t max_row;          /* longest row */
    int64_t empty_rows;
    int32_t nranks, rank;
    int64_t row_offset;       /* global index of this block's first row */
    uint64_t key;             /* history key derived from the bucketed context */
    int32_t ncandidates;
    int32_t sell_sigma;       /* σ of the prepared SELL layout (0 if not prepared) */
    double sell_fill;         /* SELL stored slots / nnz (>= 1) */
    int64_t device_bytes;     /* device memory owned by the plan */
    int64_t algorithmic_bytes;/* nnz*12 + (nrows+1)*4 + ncols*8 + nrows*8 */
    int32_t exchange;         /* resolved pepp_exchange_t */
    int64_t halo_recv;        /* ghost entries received per exchange (halo) */
    int64_t halo_send;        /* entries sent per exchange (halo) */
    double sell_col16_frac;   /* fraction of SELL chunks storing 16-bit column deltas */
    uint64_t prior_key;       /* context key the cold-start prior came from (0 = none) */
    double sell_stencil_frac; /* fraction of SELL chunks stored as stencil (one offset per slot per chunk) */
    int32_t overlap;          /* 1 = NEXT_INPUT calls overlap the halo exchange with the interior rows */
    int64_t overlap_head;     /* rows [0, overlap_head) and [nrows - overlap_tail, nrows) are computed */
    int64_t overlap_tail;     /*   before the exchange starts (0 / 0 when overlap == 0) */
    int32_t predicted;        /* candidates with a prediction from opts.predict (0 = none / no function) */
    double sell_constval_frac;/* fraction of SELL chunks stored as a pattern-table id (compress_values) */
    int32_t p2p_buffers;      /* symmetric buffers registered by pepp_spmv_p2p_buffers (0 = none) */
    int64_t sell_long_rows;   /* hybrid SELL: rows longer than sell_cap summed by the segmented
                                 long-row kernel instead of the SELL layout (0 = none) */
    int64_t sell_cap;         /* hybrid SELL cap: max(64, min(share, 8 x mean)), share = one warp's
                                 part of the SELL work = (nnz/32 + 4 x chunks) / warps of one
                                 resident wave; rows up to 1024 long above it: one warp each,
                                 longer: 4096-entry segments */
    int32_t dist_candidates;  /* distribution candidates (P', exchange) timed (0 = none: nranks == 1 or
                                 dist_select = 0) — pepp_spmv_dist_stats lists them */
    int32_t dist_nparts;      /* chosen P' for PEPP_Y_NEXT_INPUT calls (nranks when not selected) */
    int32_t dist_exchange;    /* chosen exchange for PEPP_Y_NEXT_INPUT calls (PEPP_X_P2P when the
                                 registered buffers' fused push won) */
    int32_t dist_repl_nparts; /* chosen P' for PEPP_Y_REPLICATED calls (allgather) */
    double dist_probe_ms;     /* wall time the plan-time timing of the candidates took */
    double sell_ptile_frac;   /* fraction of SELL chunks in tiles (σ = 1): runs of stencil chunks
                                 (pattern chunks with compress_values, else stencil-list chunks whose
                                 values stream) computed from x ranges and values bulk-copied into
                                 shared memory (sell_tile_kernel) when x and y are 16-byte aligned */
    int64_t sell_tile_multiline; /* multi-line pattern tiles (grid stencils: K tiles D rows apart
                                 loading their K + W x lines once each; 0 = none) */
} pepp_plan_info_t;

typedef struct pepp_spmv_plan_s pepp_spmv_plan_t;  /* opaque plan (C forbids a typedef and a function sharing the name pepp_spmv_plan) */

/* ---- core calls ----------------------------------------------------- */

/* Human-readable name of a status code (static storage; never NULL). */
const char* pepp_status_str(pepp_status_t s);

/* Fill *opts with the defaults documented above. The composition tool's
   global switches (the paper's disableImpls, P@16687, and useHistoryModels,
   "per component or global", P@28058) can be given as environment defaults,
   read here only (fields a caller sets afterwards win — the per-component
   form): PEPP_VARIANT = comma list of csr_vector, merge_path, sell,
   csr_stream, panel (the allowed variants -> variant_mask; no known name =
   all); PEPP_USE_HISTORY = 0 / 1 (use_history); PEPP_HISTORY_PATH = file
   (history_path; the string must stay in the environment while the options
   are used). */
void pepp_spmv_opts_default(pepp_spmv_opts_t* opts);

/* Build a plan for A on opts->device. Copies A; the plan owns all device
   memory it allocates. Host arrays of A are only read during the call;
   pageable ones of 64 MB or more are staged through a process-wide pool of
   pinned buffers (16 x 16 MB, allocated on first use and kept for the
   process) by 8 host threads. Collective over ranks when opts->nranks > 1 (every
   rank must call it with its own row block). On error *out is NULL.
   Errors: PEPP_E_INVALID (NULL args, broken CSR invariants, bad options),
   PEPP_E_CUDA (no device / CUDA failure), PEPP_E_NOMEM, PEPP_E_NCCL,
   PEPP_E_UNSUPPORTED (nnz >= 2^31 in one block, ncols >= 2^31). */
pepp_status_t pepp_spmv_plan(const pepp_csr_t* A, const pepp_spmv_opts_t* opts,
                             pepp_spmv_plan_t** out);

/* The choice pepp_spmv_exec(force = NULL) would make now. Host only: no
   device synchronisation; harvests finished timing events without blocking.
   Budget: < 2 µs (the paper's runtime task overhead, P@40366). */
pepp_status_t pepp_spmv_select(pepp_spmv_plan_t* p, pepp_choice_t* out);

/* y = A·x for this plan's rows, enqueued on `stream` (cudaStream_t; NULL =
   legacy default stream) and returned without waiting (asynchronous, P@17990).
   x: READ, device, ncols entries (global length), not modified, must not
      overlap y.
   y: WRITE, device, global-length buffer (row_bounds[nranks] entries when
      partitioned, else nrows); this block's rows land at
      y[row_offset .. row_offset+nrows). With PEPP_Y_NEXT_INPUT /
      PEPP_Y_REPLICATED the exchange then fills ghost / all entries from the
      other ranks (NCCL, same stream). Entries not covered by `flags` are
      left untouched.
   force: NULL = automatic selection; else force->variant/param (and, when
      partitioned, force->exchange and force->nparts: P' > 0 and < nranks runs
      the call on ranks 0..P'-1 as a distribution candidate does; nparts <= 0
      or == nranks means this rank's own block) select the implementation.
   used: optional; receives the choice that ran (launches = this library's
      kernels the call enqueued).
   Some plans also use their own second stream inside a call (the genlist
   walk beside the stencil-list kernel, the overlapped halo): it forks from
   `stream` after the caller's queued work and joins back before the call's
   last operation on `stream`, so completion of `stream` means y is written.
   Errors: PEPP_E_INVALID (NULL / aliasing / unknown forced variant or
   masked-out variant), PEPP_E_CUDA, PEPP_E_NCCL, PEPP_E_STATE (exchange
   requested on an unpartitioned plan is fine and a no-op; a plan in a sticky
   error state returns its error). */
pepp_status_t pepp_spmv_exec(pepp_spmv_plan_t* p, const void* x, void* y, int flags,
                             void* stream, const pepp_choice_t* force, pepp_choice_t* used);

/* The exchange step alone: make this rank's rows of y
   usable by the other ranks' next call, on `stream`. flags as in
   pepp_spmv_exec (PEPP_Y_NEXT_INPUT: the plan's exchange, halo or
   allgatherv; PEPP_Y_REPLICATED: allgatherv). y: READWRITE device buffer,
   global length; own rows are read, other rows written. exec(flags) ==
   exec(PEPP_Y_LOCAL) followed by exchange(flags). A no-op when nranks == 1.
   Errors: PEPP_E_INVALID, PEPP_E_NCCL, PEPP_E_CUDA. */
pepp_status_t pepp_spmv_exchange(pepp_spmv_plan_t* p, void* y, int flags, void* stream);

/* Symmetric buffers for the fused peer-memory halo (PEPP_X_P2P).
   The paper partitions a component call into sub-tasks whose outputs are
   concatenated (§IV-F P@27330–28000) and overlaps their communication with
   computation; on B200s joined by NVSwitch the concatenation can be done by
   the kernel that produces the rows: it stores them into the neighbours'
   memory directly (SURVEY §8(e) "Stretch": fuse the ghost push into the
   SpMV). Collective over the plan's ranks (every rank calls it with the
   same nbuf). Allocates nbuf (1..4) device buffers of row_bounds[nranks]
   elements of the plan's value type (zeroed) plus a small signal block,
   exports them with CUDA IPC, all-gathers the handles over the plan's
   communicator and maps the buffers of the ranks this rank sends to
   (cudaIpcMemLazyEnablePeerAccess). bufs: WRITE, host array of nbuf
   pointers that receive this rank's buffers (owned by the plan, valid until
   pepp_spmv_destroy, which is then collective too).
   Afterwards a pepp_spmv_exec(flags = PEPP_Y_NEXT_INPUT, force = NULL) whose
   y is bufs[i] — the same i on every rank, every rank making the same
   sequence of such calls — computes the interior rows on `stream` and, on
   the plan's side stream, runs ONE kernel that computes the head / tail rows,
   writes them to y and to the peers' bufs[i], and signals / waits on the
   peers (protocol in kernels.cuh, halo_push_kernel); the call's stream work
   completes when own rows and every ghost are in y, as with the NCCL halo.
   Rows of this block outside the ghosts a peer reads may also be written
   into that peer's buffer (with their correct values). Calls with any other
   y use the NCCL exchange. Boundary rows are summed in the oracle's order
   (no FMA). Readiness flows from each receiver to its senders and data from
   senders to receivers, so the send and receive peer sets may differ
   (nonsymmetric matrices). Requires nranks > 1, the halo exchange and, on
   every rank that sends rows, the head / interior / tail split
   (pepp_plan_info_t.overlap == 1; a rank that sends nothing computes its
   whole block on `stream` and only signals). The ranks agree first (one
   max-reduce): if any rank cannot take part, EVERY rank returns
   PEPP_E_UNSUPPORTED and the plan stays usable with the NCCL halo. A CUDA
   failure on any rank (IPC export or peer mapping) is also agreed on: every
   rank returns PEPP_E_CUDA, the partial registration is undone and the plan
   stays usable with the NCCL halo (callers fall back; bench.py does). Only
   a failing collective (PEPP_E_NCCL) leaves the plan in a sticky error.
   Test hook: environment PEPP_FAULT_P2P_EXPORT=<rank> makes that rank's
   export fail (fault injection for the fallback test; no other effect).
   PEPP_E_STATE if already registered. A peer that stops calling makes the
   waiting kernel give up after 20 s and the plan's next call return
   PEPP_E_NCCL. Errors: PEPP_E_INVALID, PEPP_E_CUDA (IPC unavailable),
   PEPP_E_NCCL, PEPP_E_NOMEM. */
pepp_status_t pepp_spmv_p2p_buffers(pepp_spmv_plan_t* p, int32_t nbuf, void** bufs);

/* Distribution candidates of a partitioned plan (opts.dist_select; the
   runtime's choice of "which implementation/device to use" from history
   and data-transfer cost, §V-D P@38827; §8(a) a4): for each i < *n (up to
   cap): nparts[i] = P', exchange[i] = pepp_exchange_t (the last entry is
   PEPP_X_P2P once pepp_spmv_p2p_buffers registered buffers), agreed_us[i] =
   the max-over-ranks mean time of one PEPP_Y_NEXT_INPUT call the ranks
   agreed on (0 if never timed). nparts / exchange / agreed_us: WRITE, host,
   cap entries each, or NULL; *n: WRITE, the total. Host only.
   PEPP_E_INVALID on NULL p or n, negative cap. */
pepp_status_t pepp_spmv_dist_stats(const pepp_spmv_plan_t* p, int32_t cap, int32_t* nparts, int32_t* exchange,
                                   double* agreed_us, int32_t* n);

/* Host-buffer entry point (the paper's measurement setting, where operand
   transfers are part of the call: Fig. 5 "communication overhead of copying
   data back and forth to device memory is also included", P@35591–35720).
   Copies x_host (READ, host, ncols entries; pinned memory gives full PCIe /
   C2C speed) into a plan-owned device buffer, runs `iterations` >= 1 calls
   x_{k+1} = A·x_k (iterations > 1 needs a square global matrix: ncols ==
   global rows, reading A11) with the exchange `flags` asks for
   (PEPP_Y_NEXT_INPUT is implied between iterations when partitioned), then
   copies the final y into y_host (WRITE, host, global-length; all global rows
   with PEPP_Y_REPLICATED, else only this rank's rows are written) and waits
   for completion on `stream`.
   The plan-owned device buffers are allocated on first use and kept
   ("register once", P@29208). Errors as pepp_spmv_exec. */
pepp_status_t pepp_spmv_exec_host(pepp_spmv_plan_t* p, const void* x_host, void* y_host, int32_t iterations,
                                  int flags, void* stream);

/* pepp_spmv_exec_host over `nbatch` independent right-hand sides: item k
   reads x_hosts[k] (READ, host, ncols entries) and writes y_hosts[k] (WRITE,
   host, rows as in pepp_spmv_exec_host), with `iterations` and `flags` as
   there. The transfers overlap the computation — item k+1's input copy and
   item k-1's output copy run on the copy engines while item k computes —
   the data-transfer overlap the runtime is meant to provide for
   GPU-resident operands (§IV-E, P@21908–27091; transfer-inclusive timing of
   Fig. 5, P@35591–35720). Results equal nbatch separate pepp_spmv_exec_host
   calls. Work starts after everything queued on `stream`; the call returns
   when every y_hosts[k] is written. Host buffers must be pinned for the
   copies to overlap (pageable buffers are correct, only serialised). Entries
   may repeat: output copies run in item order, so a repeated y buffer ends
   with its last item's result; a y buffer must not overlap an x buffer of
   the batch. Two slots of plan-owned device buffers (4 vectors
   of max(ncols, global rows) entries) and two copy streams are created on
   first use and kept. nbatch = 0 is a no-op; nbatch = 1 is
   pepp_spmv_exec_host. Errors: PEPP_E_INVALID (NULL arrays or entries,
   nbatch < 0, iterations < 1 or > 1 on a non-square matrix), otherwise as
   pepp_spmv_exec. */
pepp_status_t pepp_spmv_exec_host_batch(pepp_spmv_plan_t* p, int32_t nbatch, const void* const* x_hosts,
                                        void* const* y_hosts, int32_t iterations, int flags, void* stream);

/* Free everything the plan owns (device memory, events, an owned NCCL
   communicator); saves history to opts.history_path if set. Waits for the
   plan's outstanding work. NULL is a no-op. */
pepp_status_t pepp_spmv_destroy(pepp_spmv_plan_t* p);

/* ---- introspection -------------------------------------------------- */

pepp_status_t pepp_spmv_plan_info(const pepp_spmv_plan_t* p, pepp_plan_info_t* out);

/* Copy up to `cap` candidates (variant, param, exchange) into out; *n gets the total. */
pepp_status_t pepp_spmv_candidates(const pepp_spmv_plan_t* p, pepp_choice_t* out, int32_t cap, int32_t* n);

/* Block until every recorded timing is available and fold it into the history. */
pepp_status_t pepp_spmv_flush_history(pepp_spmv_plan_t* p);

/* History statistics of candidate `cand` for this plan's key. */
pepp_status_t pepp_spmv_history_stats(const pepp_spmv_plan_t* p, int32_t cand,
                                      int64_t* count, double* mean_us, double* m2);

/* ---- CUDA graphs for launch-bound calls --------------------------------
   Small matrices (BASELINE config 1: 20 K nonzeros, a few µs of work) are
   bound by launch and host overhead, like the paper's ODE solver making
   10,613 small component calls (Fig. 7, P@41298). A graph captures
   `iterations` calls once — the variant the selector would choose now, with
   its exchange — and replays them with one launch.
   mode 0 (repeat): every call computes y = A·x (same x, same y).
   mode 1 (iterate): x_{k+1} = A·x_k, ping-pong between y and `work`
   (device, same length as y; x is read only by the first call); the result
   of the last call is in y when `iterations` is odd, else in work.
   x, y, work: device buffers that must stay valid while the graph exists.
   Timing events are not recorded inside graphs (history is not updated by
   replays). Errors: PEPP_E_INVALID, PEPP_E_CUDA, PEPP_E_NCCL. */
typedef struct pepp_spmv_graph_s pepp_spmv_graph_t;
pepp_status_t pepp_spmv_graph_create(pepp_spmv_plan_t* p, const void* x, void* y, void* work,
                                     int32_t iterations, int32_t mode, int flags, void* stream,
                                     pepp_spmv_graph_t** out);
pepp_status_t pepp_spmv_graph_launch(pepp_spmv_graph_t* g, void* stream);
pepp_status_t pepp_spmv_graph_destroy(pepp_spmv_graph_t* g);

/* ---- smart containers (paper §IV-D P@20045–21195) --
   A vector whose payload may live in host memory (the master copy) and in
   device memory at the same time, with a valid / outdated state per copy.
   Copies move only when an access needs them (paper Fig. 3, P@22400–26903):
     - device access for a component call: READ or READWRITE copies host ->
       device if the device copy is outdated; WRITE-only copies nothing
       ("the first component call only writes the data and hence no copy is
       made", P@23793); any write marks the host copy outdated;
     - host access (the paper's [] operator, element-wise R/W proxies): copies
       device -> host if the host copy is outdated (also before a host write:
       "data is copied back ... before the actual operation takes place");
       a host write marks the device copy outdated.
   Fig. 3's program (write, host read, readwrite, read, read, host write)
   therefore makes 2 copies, where copying around every call makes 7.
   Access modes: */
#define PEPP_ACCESS_READ      1
#define PEPP_ACCESS_WRITE     2
#define PEPP_ACCESS_READWRITE 3
#define PEPP_DEVICE_SIMULATED (-2)  /* state machine + counters only, no CUDA (CPU tests) */

typedef struct pepp_vector_s pepp_vector_t;

/* n fp64 elements. host: the master copy (borrowed, must outlive the vector)
   or NULL to allocate one (pinned). device: CUDA ordinal, -1 = current, or
   PEPP_DEVICE_SIMULATED. The device copy is allocated on first device use.
   Errors: PEPP_E_INVALID, PEPP_E_NOMEM, PEPP_E_CUDA. */
pepp_status_t pepp_vector_create(int64_t n, double* host, int32_t device, pepp_vector_t** out);
/* Waits for outstanding device work on the vector, frees what it owns. NULL is a no-op. */
pepp_status_t pepp_vector_destroy(pepp_vector_t* v);
/* Host access with `mode`; *host receives the master copy, valid for `mode`
   on return (blocks until any device work that uses the vector completed). */
pepp_status_t pepp_vector_acquire_host(pepp_vector_t* v, int32_t mode, double** host);
/* Device access with `mode` for work the caller enqueues on `stream`; the
   needed copy (if any) is enqueued on `stream`; *dev receives the device copy
   (NULL for a simulated vector). Call pepp_vector_release_device after
   enqueueing the work. */
pepp_status_t pepp_vector_acquire_device(pepp_vector_t* v, int32_t mode, void* stream, double** dev);
/* Records the end of the device work on `stream` that used the vector. */
pepp_status_t pepp_vector_release_device(pepp_vector_t* v, void* stream);
/* Copies made so far (host->device, device->host) and bytes moved. */
pepp_status_t pepp_vector_counters(const pepp_vector_t* v, int64_t* h2d, int64_t* d2h, int64_t* bytes);
/* Current state: 1 = that copy is valid. */
pepp_status_t pepp_vector_state(const pepp_vector_t* v, int32_t* host_valid, int32_t* device_valid);
/* A READWRITE component on a vector: v = alpha * v on the device (stream-ordered). */
pepp_status_t pepp_vector_scale(pepp_vector_t* v, double alpha, void* stream);
/* y = A·x through containers: x READ, y WRITE (see pepp_spmv_exec for flags,
   force, used). x and y must be distinct vectors of length ncols / global rows.
   Containers hold fp64: an fp32 plan returns PEPP_E_UNSUPPORTED. */
pepp_status_t pepp_spmv_exec_vec(pepp_spmv_plan_t* p, pepp_vector_t* x, pepp_vector_t* y, int flags,
                                 void* stream, const pepp_choice_t* force, pepp_choice_t* used);

/* ---- host-only utilities (no GPU needed) ---------------------------- */

/* nnz-balanced contiguous row blocks (reading A9; P@27578):
   bounds[p] = min{ r : row_ptr[r] - first >= ceil(p*nnz/nparts) } for
   0 < p < nparts, bounds[0] = 0, bounds[nparts] = nrows.
   row_ptr: READ host [nrows+1]; bounds: WRITE host [nparts+1]. */
pepp_status_t pepp_partition_rows(const int64_t* row_ptr, int64_t nrows, int64_t first,
                                  int32_t nparts, int64_t* bounds);

/* Ghost (halo) columns of one row block: the sorted distinct columns of
   col_idx[0..nnz) that lie outside [row_bounds[rank], row_bounds[rank+1]),
   grouped by owning rank. counts: WRITE [nranks] (count per owner; own rank
   gets 0). ghosts: WRITE, capacity `cap` entries, sorted ascending (so
   grouped by owner); *total gets the number of ghosts (may exceed cap, in
   which case only counts/total are valid). Host memory only. */
pepp_status_t pepp_halo_ghosts(const int32_t* col_idx, int64_t nnz, int32_t nranks, int32_t rank,
                               const int64_t* row_bounds, int64_t* counts, int32_t* ghosts,
                               int64_t cap, int64_t* total);

/* ---- history / selector object (host only; the plan embeds one) ------ */
/* A history table keyed by (context key, candidate id) with Welford
   count / mean / M2 of measured times — the runtime's "performance history"
   (P@10254). Exposed so the selection policy is testable without a GPU
   (inject times with pepp_history_record). */
typedef struct pepp_history pepp_history;

pepp_status_t pepp_history_create(pepp_history** out);
pepp_status_t pepp_history_destroy(pepp_history* h);
pepp_status_t pepp_history_record(pepp_history* h, uint64_t key, int32_t cand, double us);
pepp_status_t pepp_history_stats(const pepp_history* h, uint64_t key, int32_t cand,
                                 int64_t* count, double* mean_us, double* m2);
/* Policy (reading A10): calibration runs in rounds r = 1..min_samples —
   the lowest eligible candidate with fewer than r records is returned with
   *calibrating = 1, except that a candidate whose samples already average
   more than 4x the best mean seen so far is not sampled again (early
   abandonment: one sample rules it out). When every candidate is
   calibrated or abandoned, return argmin mean time, ties within 1 % going
   to the lower index, *calibrating = 0. *predicted_us = that candidate's
   mean. (pepp_spmv_exec applies the same policy and also counts timed calls
   still in flight.) */
pepp_status_t pepp_history_select(const pepp_history* h, uint64_t key, int32_t ncand,
                                  const uint8_t* eligible, int32_t min_samples,
                                  int32_t* cand, int32_t* calibrating, double* predicted_us);
/* Distribution choice policy (§8(a) a4, P and exchange; host only, the
   rule pepp_spmv_plan applies after its NCCL max-reduce): means is
   [nranks][nd] row-major, each rank's own measured mean time per candidate;
   a partitioned call takes as long as its slowest rank, so candidate d's
   agreed time is max over ranks of means[r][d]; *choice = argmin of the
   agreed times over eligible candidates (eligible NULL = all; a candidate
   with agreed time 0 or Inf is skipped), ties within 1 % going to the lower
   index (reading A10). agreed: optional [nd] output. PEPP_E_INVALID on NULL
   or negative / NaN input, PEPP_E_STATE if nothing is eligible. */
pepp_status_t pepp_dist_choose(int32_t nranks, int32_t nd, const double* means, const uint8_t* eligible,
                               int32_t* choice, double* agreed);

/* Cold-start prior (static composition from recorded runs, P@10069, P@10489):
   the nearest context key to `key` (L1 distance over the bucket fields of
   pepp_context_key; same rank count) that has samples for some of the
   candidate ids ids[0..n); prior[c] = that key's mean for ids[c] (-1 if it
   has none). PEPP_E_STATE if no such key exists. A plan with an unseen key
   uses this prior (from a loaded history_path) to calibrate the predicted
   best candidate first and to skip candidates predicted > 4x slower. */
pepp_status_t pepp_history_prior(const pepp_history* h, uint64_t key, int32_t n, const int32_t* ids,
                                 double* prior, uint64_t* from_key);
pepp_status_t pepp_history_save(const pepp_history* h, const char* path);
pepp_status_t pepp_history_load(pepp_history* h, const char* path);

/* Context key of a row-pointer array (host): bucketed (log2 rows, log2 nnz,
   mean row length, CV, nparts) plus the kernel instance — the "context
   instance" used as history key (§III P@9781). `instance` is a bit set:
   PEPP_KEY_F32 for an fp32 plan, PEPP_KEY_COMPRESS for a plan built with
   opts.compress_values = 1 (both select different kernels, so their timings
   must not be mixed with the fp64 / value-streaming plan's). A cold-start
   prior (pepp_history_prior) is only taken from a key with the same rank
   count and instance. */
#define PEPP_KEY_F32      0x1
#define PEPP_KEY_COMPRESS 0x2
#define PEPP_KEY_DIST     0x4   /* the distribution (P', exchange) records of a partitioned plan */
uint64_t pepp_context_key(int64_t nrows, int64_t ncols, int64_t nnz, double cv, int32_t nparts, int32_t instance);

/* NCCL bootstrap helper: write a fresh 128-byte ncclUniqueId into id_out
   (NCCL is loaded on demand with dlopen; PEPP_E_NCCL if unavailable). */
pepp_status_t pepp_nccl_unique_id(void* id_out);

/* NCCL self-test on `device` (-1 = current): a one-rank communicator runs
   every NCCL call the partitioned path makes — grouped ncclSend/ncclRecv to
   itself (int32, int64, fp32, fp64), in-place ncclBroadcast, ncclAllReduce
   (max) — and checks the bytes that arrive. Verifies that the NCCL found at
   run time (dlopen: PEPP_NCCL_LIB, else the copy already loaded, else the
   system one) matches the calling convention this library was built against.
   PEPP_OK, PEPP_E_NCCL (unavailable, an NCCL error, or wrong data), or
   PEPP_E_CUDA. Synchronous; allocates and frees its own buffers. */
pepp_status_t pepp_nccl_selftest(int32_t device);

/* Text of the last CUDA failure that made a call on this thread return
   PEPP_E_CUDA: the CUDA error string, the failing runtime call and its
   source line ("" if none yet). Thread-local, static storage, never NULL. */
const char* pepp_last_error(void);

/* ABI version (PEPP_ABI_VERSION) of the loaded library. */
int32_t pepp_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PEPP_SPMV_H */
