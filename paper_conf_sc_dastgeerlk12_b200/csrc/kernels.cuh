// kernels.cuh — sm_100a kernels of the SpMV hot path (y = A·x over CSR, fp64).
//
// The paper's GPU variant was a library call into CUSP on Fermi / GT200
// (PAPER.md P@33595, P@35591); these three hand-written variants replace it
// (implementation variants of one interface, §II P@4772). SpMV is not a dense
// contraction, so no tensor cores: every kernel is bound by HBM streaming of
// val (8 B) + col (4 B) per nonzero; the design levers are
// coalescing, 128-bit loads, bytes in flight, and keeping x in L2.
//
// Device CSR layout (built by plan.cu):
//   rp[0..nrows]   int32, rp[i] = row_ptr[i] - first + pad, pad = first mod 4,
//                  so the 4-element alignment of every entry equals its
//                  alignment in the caller's global array (partition
//                  invariance).
//   col[], val[]   pad leading zeros + nnz entries + >= 4 trailing zeros
//                  (val = 0, col = 0), 16-B aligned, so aligned 4-groups
//                  never read out of bounds.
//   x              global length; y points at this block's first row.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <type_traits>

namespace pepp {
namespace k {

// ----------------------------------------------------------------- loads
// Streaming loads for the matrix (read exactly once per call): non-coherent
// path, no L1 allocation, L2 evict-first policy (createpolicy) so that x
// keeps its L2 residency. (On sm_100a the bare .L2::evict_first qualifier is
// only accepted on 256-bit loads; the cache_hint form works for every width.)
// Not `volatile`: the matrix is read-only during a launch, and volatile asm
// would pin the loads in program order and stop ptxas from batching them.
__device__ __forceinline__ uint64_t evict_first_policy() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ int4 ld_stream_i4(const int* p, uint64_t pol) {
    int4 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ double2 ld_stream_d2(const double* p, uint64_t pol) {
    double2 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;"
                 : "=d"(r.x), "=d"(r.y) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ double ld_stream_d(const double* p, uint64_t pol) {
    double r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(r) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ int ld_stream_i16(const int16_t* p, uint64_t pol) {
    int r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s16 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ int ld_stream_i(const int* p, uint64_t pol) {
    int r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ float ld_stream_f(const float* p, uint64_t pol) {
    float r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(r) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ float4 ld_stream_f4(const float* p, uint64_t pol) {
    float4 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
        : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p), "l"(pol));
    return r;
}
// value-type generic forms (T = double for the fp64 path, float for the
// fp32 instance of the paper's `float` signature)
__device__ __forceinline__ double ld_stream_v(const double* p, uint64_t pol) { return ld_stream_d(p, pol); }
__device__ __forceinline__ float ld_stream_v(const float* p, uint64_t pol) { return ld_stream_f(p, pol); }
// four consecutive values starting at a 4-element-aligned position (16 B for
// float: one load; 32 B for double: two)
__device__ __forceinline__ void ld_stream_4(const double* p, uint64_t pol, double v[4]) {
    const double2 a = ld_stream_d2(p, pol), b = ld_stream_d2(p + 2, pol);
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
}
__device__ __forceinline__ void ld_stream_4(const float* p, uint64_t pol, float v[4]) {
    const float4 a = ld_stream_f4(p, pol);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
}
// x gather: read-only path, cached in L1 and L2 (reused across rows)
template <typename T>
__device__ __forceinline__ T ld_x(const T* __restrict__ x, int c) { return __ldg(x + c); }
// same gather as volatile asm: a run of these is issued back-to-back in
// program order (ptxas may not interleave the consumers between them)
__device__ __forceinline__ double ld_x_ordered(const double* __restrict__ x, int c) {
    double r;
    asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(r) : "l"(x + c));
    return r;
}
__device__ __forceinline__ float ld_x_ordered(const float* __restrict__ x, int c) {
    float r;
    asm volatile("ld.global.nc.f32 %0, [%1];" : "=f"(r) : "l"(x + c));
    return r;
}

// =====================================================================
// Variant 0: vector-CSR with TPR lanes per row (TPR in {2,4,8,16,32}).
// Each lane walks aligned 4-element groups of its row with stride TPR:
// one int4 of columns + two double2 of values per group (3 x 16-B loads),
// entries outside the row are masked. Partial sums are combined with a
// __shfl_xor_sync butterfly over the TPR lanes. The row loop is warp-
// uniform (all 32 lanes iterate together) so full-mask shuffles are legal.
// =====================================================================
template <int TPR, int BLOCK, typename T>
__global__ void __launch_bounds__(BLOCK) csr_vector_kernel(int nrows, const int* __restrict__ rp,
                                                           const int* __restrict__ col,
                                                           const T* __restrict__ val,
                                                           const T* __restrict__ x,
                                                           T* __restrict__ y) {
    static_assert(TPR >= 1 && TPR <= 32 && (TPR & (TPR - 1)) == 0, "TPR must be a power of two <= 32");
    constexpr int RPW = 32 / TPR;                 // rows per warp per step
    const int lane = threadIdx.x & 31;
    const int sub = lane & (TPR - 1);             // lane within the row group
    const int grp = lane / TPR;                   // row group within the warp
    const int warp = (blockIdx.x * BLOCK + threadIdx.x) >> 5;
    const int nwarps = (gridDim.x * BLOCK) >> 5;
    const uint64_t pol = evict_first_policy();

    // the next row's [s, e) is prefetched while the current row's entries
    // are in flight (one dependent round trip less per row)
    const int64_t step = (int64_t)nwarps * RPW;
    int64_t base = (int64_t)warp * RPW;
    int sn = 0, en = 0;
    if (base + grp < nrows) {
        sn = __ldg(rp + base + grp);
        en = __ldg(rp + base + grp + 1);
    }
    for (; base < nrows; base += step) {
        const int64_t row = base + grp;
        const int s = sn, e = en;
        if (row + step < nrows) {
            sn = __ldg(rp + row + step);
            en = __ldg(rp + row + step + 1);
        }
        T acc = T(0);
        const int g_end = (e + 3) >> 2;
        int g = (s >> 2) + sub;
        // two groups per iteration: up to 6 independent 16-B loads in flight per lane
        for (; g + TPR < g_end; g += 2 * TPR) {
            const int k0 = g << 2, k1 = (g + TPR) << 2;
            const int4 c0 = ld_stream_i4(col + k0, pol);
            T v0[4], v1[4];
            ld_stream_4(val + k0, pol, v0);
            const int4 c1 = ld_stream_i4(col + k1, pol);
            ld_stream_4(val + k1, pol, v1);
            // group g is not the row's last group: only its head can precede s
            if (k0 + 0 >= s) acc = fma(v0[0], ld_x(x, c0.x), acc);
            if (k0 + 1 >= s) acc = fma(v0[1], ld_x(x, c0.y), acc);
            if (k0 + 2 >= s) acc = fma(v0[2], ld_x(x, c0.z), acc);
            if (k0 + 3 >= s) acc = fma(v0[3], ld_x(x, c0.w), acc);
            // group g+TPR starts after s: only its tail can pass e
            if (k1 + 0 < e) acc = fma(v1[0], ld_x(x, c1.x), acc);
            if (k1 + 1 < e) acc = fma(v1[1], ld_x(x, c1.y), acc);
            if (k1 + 2 < e) acc = fma(v1[2], ld_x(x, c1.z), acc);
            if (k1 + 3 < e) acc = fma(v1[3], ld_x(x, c1.w), acc);
        }
        if (g < g_end) {
            const int k0 = g << 2;
            const int4 c0 = ld_stream_i4(col + k0, pol);
            T v0[4];
            ld_stream_4(val + k0, pol, v0);
            if (k0 + 0 >= s && k0 + 0 < e) acc = fma(v0[0], ld_x(x, c0.x), acc);
            if (k0 + 1 >= s && k0 + 1 < e) acc = fma(v0[1], ld_x(x, c0.y), acc);
            if (k0 + 2 >= s && k0 + 2 < e) acc = fma(v0[2], ld_x(x, c0.z), acc);
            if (k0 + 3 >= s && k0 + 3 < e) acc = fma(v0[3], ld_x(x, c0.w), acc);
        }
#pragma unroll
        for (int off = TPR / 2; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (sub == 0 && row < nrows) y[row] = acc;
    }
}

// =====================================================================
// Variant 2: SELL-C-σ, C = 32. Chunk c holds the 32 (sorted) rows
// [32c, 32c+32): slot j of lane l is at chunk_ptr[c] + 32*j + l, so a warp
// reads 256 contiguous bytes of values and 128 of columns per slot.
// chunk_len[c] >= 0: every row of the chunk has exactly that many entries
// (no per-row length is read); chunk_len[c] < 0: -chunk_len[c] slots and
// each lane masks the slots beyond its own row length rowlen[32c+l] (no
// padding arithmetic, so Inf/NaN in x behave exactly as in the CSR
// definition). perm maps sorted position -> original row (NULL when σ = 1).
// The kernel is latency-bound at one chunk per warp, so each chunk's slots
// are loaded in batches of up to 8 (all column and value loads, then all x
// gathers, then the FMAs) with an exactly-sized tail batch, and the next
// chunk's metadata is prefetched (tools/experiments/sell_probe.cu: 830 ->
// 771 us on config 4). The grid is one resident wave (SMs x occupancy).
// =====================================================================
// Chunk descriptor bits in chunk_len[c]: low 28 bits = slots in the chunk;
// bit 30 = masked (rows of the chunk have different lengths: read rowlen);
// bit 29 = 16-bit columns (col16 holds col - row, row = the original index of
// the lane's row; every delta of the chunk fits in int16);
// bit 28 = stencil chunk (every lane has the same column offsets relative to
// its row: soff[chunk_ptr[c]/32 + j] holds the offset of slot j once for the
// whole chunk — a per-chunk diagonal (DIA) layout; no column stream at all).
constexpr int kSellMasked = 1 << 30;
constexpr int kSellCol16 = 1 << 29;
constexpr int kSellStencil = 1 << 28;
constexpr int kSellPattern = 1 << 27;    // chunk = one entry of the plan's pattern table (offsets + values)
constexpr int kSellLenMask = (1 << 27) - 1;
enum { kIdx32 = 0, kIdx16 = 1, kIdxStencil = 2 };

// N slots of one chunk, loads issued unconditionally (all N exist for every
// lane) before the first FMA; the per-lane row length only masks the FMA.
// IDX: kIdx32 columns; kIdx16 int16 deltas from the lane's row index `row0`;
// kIdxStencil one offset per slot for the whole chunk (lane j's `offl`).
template <int N, int IDX, typename T>
__device__ __forceinline__ T sell_slots(const T* __restrict__ val, const int* __restrict__ col,
                                        const int16_t* __restrict__ col16, int offl,
                                        int row0, const T* __restrict__ x, int64_t base, int j0,
                                        int len, T acc, uint64_t pol) {
    T v[N];
    int c[N];
#pragma unroll
    for (int u = 0; u < N; ++u)
        c[u] = IDX == kIdxStencil ? row0 + __shfl_sync(0xffffffffu, offl, j0 + u)   // lane j holds slot j's offset
             : IDX == kIdx16      ? row0 + ld_stream_i16(col16 + base + (int64_t)(j0 + u) * 32, pol)
                                  : ld_stream_i(col + base + (int64_t)(j0 + u) * 32, pol);
#pragma unroll
    for (int u = 0; u < N; ++u) v[u] = ld_stream_v(val + base + (int64_t)(j0 + u) * 32, pol);
    T xv[N];
#pragma unroll
    for (int u = 0; u < N; ++u) xv[u] = ld_x(x, c[u]);
#pragma unroll
    for (int u = 0; u < N; ++u)
        if (j0 + u < len) acc = fma(v[u], xv[u], acc);
    return acc;
}

// Two unmasked chunks of N slots each and one format (a warp's chunks i and i+1):
// every load of both issued before the first FMA — twice the bytes in flight
// of one chunk. Per row the same products and the same slot-order sums as
// sell_slots: results are bit-identical. Measured on config 4: fp64 605 ->
// 587 µs (DRAM 99 % of the copy peak), fp32 420 -> 436 µs, so it is compiled
// into the fp64 kernel only.
template <int N, int IDX, typename T>
__device__ __forceinline__ void sell_pair(const T* __restrict__ val, const int* __restrict__ col,
                                          const int16_t* __restrict__ col16, const T* __restrict__ x, int offa,
                                          int rowa, int64_t basea, int offb, int rowb, int64_t baseb, T& acca,
                                          T& accb, uint64_t pol) {
    int ca[N], cb[N];
    T va[N], vb[N], xa[N], xb[N];
#pragma unroll
    for (int u = 0; u < N; ++u) {
        if (IDX == kIdxStencil) {
            ca[u] = rowa + __shfl_sync(0xffffffffu, offa, u);
            cb[u] = rowb + __shfl_sync(0xffffffffu, offb, u);
        } else if (IDX == kIdx16) {
            ca[u] = rowa + ld_stream_i16(col16 + basea + (int64_t)u * 32, pol);
            cb[u] = rowb + ld_stream_i16(col16 + baseb + (int64_t)u * 32, pol);
        } else {
            ca[u] = ld_stream_i(col + basea + (int64_t)u * 32, pol);
            cb[u] = ld_stream_i(col + baseb + (int64_t)u * 32, pol);
        }
    }
#pragma unroll
    for (int u = 0; u < N; ++u) {
        va[u] = ld_stream_v(val + basea + (int64_t)u * 32, pol);
        vb[u] = ld_stream_v(val + baseb + (int64_t)u * 32, pol);
    }
#pragma unroll
    for (int u = 0; u < N; ++u) { xa[u] = ld_x(x, ca[u]); xb[u] = ld_x(x, cb[u]); }
    acca = T(0);
    accb = T(0);
#pragma unroll
    for (int u = 0; u < N; ++u) { acca = fma(va[u], xa[u], acca); accb = fma(vb[u], xb[u], accb); }
}

template <int IDX, typename T>
__device__ __forceinline__ void sell_pair_len(int n, const T* __restrict__ val, const int* __restrict__ col,
                                              const int16_t* __restrict__ col16, const T* __restrict__ x, int offa,
                                              int rowa, int64_t basea, int offb, int rowb, int64_t baseb, T& a,
                                              T& b, uint64_t pol) {
    switch (n) {
    case 1: sell_pair<1, IDX, T>(val, col, col16, x, offa, rowa, basea, offb, rowb, baseb, a, b, pol); break;
    case 2: sell_pair<2, IDX, T>(val, col, col16, x, offa, rowa, basea, offb, rowb, baseb, a, b, pol); break;
    case 3: sell_pair<3, IDX, T>(val, col, col16, x, offa, rowa, basea, offb, rowb, baseb, a, b, pol); break;
    case 4: sell_pair<4, IDX, T>(val, col, col16, x, offa, rowa, basea, offb, rowb, baseb, a, b, pol); break;
    case 5: sell_pair<5, IDX, T>(val, col, col16, x, offa, rowa, basea, offb, rowb, baseb, a, b, pol); break;
    case 6: sell_pair<6, IDX, T>(val, col, col16, x, offa, rowa, basea, offb, rowb, baseb, a, b, pol); break;
    case 7: sell_pair<7, IDX, T>(val, col, col16, x, offa, rowa, basea, offb, rowb, baseb, a, b, pol); break;
    default: sell_pair<8, IDX, T>(val, col, col16, x, offa, rowa, basea, offb, rowb, baseb, a, b, pol); break;
    }
}

#ifndef PEPP_SELL_PAIR_ALL
#define PEPP_SELL_PAIR_ALL 0   // also pair 16- / 32-bit column chunks (experiment)
#endif

#ifndef PEPP_SELL_PAIR_F64
#define PEPP_SELL_PAIR_F64 0   // pairing helped the general walk on config 4 (605 -> 587 us) but costs 9-slot banded chunks 11 % (200 -> 223 us, tools/gpu_banded.sh); the stencil list now carries config 4
#endif
#ifndef PEPP_SELL_PAIR_F32
#define PEPP_SELL_PAIR_F32 0   // fp32 420 -> 436 us: off
#endif
#ifndef PEPP_SELL_PAIR_SORTED
#define PEPP_SELL_PAIR_SORTED 0   // pair equal chunks in σ > 1 walks: config 3 358 -> 373 us, skew 249 -> 268 us (84 vs fewer registers): off
#endif
template <typename T>
constexpr bool sell_pairs() { return std::is_same<T, float>::value ? PEPP_SELL_PAIR_F32 : PEPP_SELL_PAIR_F64; }

template <int IDX, typename T>
__device__ __forceinline__ T sell_chunk(const T* __restrict__ val, const int* __restrict__ col,
                                        const int16_t* __restrict__ col16, int offl, int row0,
                                        const T* __restrict__ x, int64_t base, int clen, int len, uint64_t pol) {
    T acc = T(0);
    int j = 0;
    // whole blocks of 8 slots, then one exactly-sized tail (warp-uniform switch)
    for (; j + 8 <= clen; j += 8) acc = sell_slots<8, IDX, T>(val, col, col16, offl, row0, x, base, j, len, acc, pol);
    switch (clen - j) {
    case 1: acc = sell_slots<1, IDX, T>(val, col, col16, offl, row0, x, base, j, len, acc, pol); break;
    case 2: acc = sell_slots<2, IDX, T>(val, col, col16, offl, row0, x, base, j, len, acc, pol); break;
    case 3: acc = sell_slots<3, IDX, T>(val, col, col16, offl, row0, x, base, j, len, acc, pol); break;
    case 4: acc = sell_slots<4, IDX, T>(val, col, col16, offl, row0, x, base, j, len, acc, pol); break;
    case 5: acc = sell_slots<5, IDX, T>(val, col, col16, offl, row0, x, base, j, len, acc, pol); break;
    case 6: acc = sell_slots<6, IDX, T>(val, col, col16, offl, row0, x, base, j, len, acc, pol); break;
    case 7: acc = sell_slots<7, IDX, T>(val, col, col16, offl, row0, x, base, j, len, acc, pol); break;
    default: break;
    }
    return acc;
}

// Pattern table (value + index compression): chunks whose 32 rows share
// their column offsets AND whose every slot holds one bitwise-identical value
// (constant-coefficient stencils) are stored as an id into this table, passed
// by value as a kernel parameter (constant bank: uniform LDC reads, no
// memory stream). The chunk reads only x and writes y.
constexpr int kSellMaxPatterns = 32;
#ifndef PEPP_PAT_MAXLEN
#define PEPP_PAT_MAXLEN 16   // slots of a pattern-table entry (9-point / 3-D stencils up to 16 slots)
#endif
constexpr int kSellMaxPatternLen = PEPP_PAT_MAXLEN;
template <typename T>
struct SellPatterns {
    int len[kSellMaxPatterns];
    int off[kSellMaxPatterns][kSellMaxPatternLen];
    T val[kSellMaxPatterns][kSellMaxPatternLen];
};

template <int N, typename T>
__device__ __forceinline__ T sell_pattern_slots(const SellPatterns<T>& pt, int pid, int row0,
                                                const T* __restrict__ x) {
    int c[N];
    T xv[N];
#pragma unroll
    for (int u = 0; u < N; ++u) c[u] = row0 + pt.off[pid][u];
#pragma unroll
    for (int u = 0; u < N; ++u) xv[u] = ld_x(x, c[u]);
    T acc = T(0);
#pragma unroll
    for (int u = 0; u < N; ++u) acc = fma(pt.val[pid][u], xv[u], acc);   // slot order = the row's CSR order
    return acc;
}

#ifndef PEPP_PAT_U
#define PEPP_PAT_U 4
#endif
constexpr int kPatU = PEPP_PAT_U;   // pattern chunks per warp iteration in phase A
#ifndef PEPP_PAT_INFLIGHT
#define PEPP_PAT_INFLIGHT 20   // x gathers in flight per lane in phase A (sub-groups beyond)
#endif
#ifndef PEPP_PAT_PREFETCH
#define PEPP_PAT_PREFETCH 1   // L2 prefetch distance in groups (0 = off; 1 measured best: 265 -> 254 us on config 4)
#endif

// list entries k0, k0 + stride, ... (kPatU of them; -1 past the end)
__device__ __forceinline__ void sell_pattern_ids(const int* __restrict__ patlist, int npatc, int k0, int stride,
                                                 int (&q)[kPatU]) {
#pragma unroll
    for (int u = 0; u < kPatU; ++u) { const int kk = k0 + u * stride; q[u] = kk < npatc ? __ldg(patlist + kk) : -1; }
}

// Groups of kPatU chunks of pattern `pid` (N slots) starting at list index
// k0 (entries already in q), the next group's entries prefetched: the
// pattern is read from the parameter table once into registers (indexed LDCs
// per chunk would run on the narrow ADU pipe); all loads of the group are
// issued before the first FMA. Returns the list index of the first group that
// is not all `pid` (q then holds it), or >= npatc when the warp is done.
template <int N, typename T>
__device__ __forceinline__ int sell_pattern_run(const SellPatterns<T>& pt, int pid, const int* __restrict__ patlist,
                                             int npatc, int k0, int stride, int (&q)[kPatU], int lane,
                                             const T* __restrict__ x, T* __restrict__ y) {
    int o[N];
    T v[N];
#pragma unroll
    for (int j = 0; j < N; ++j) { o[j] = pt.off[pid][j]; v[j] = pt.val[pid][j]; }
    for (; k0 < npatc; k0 += kPatU * stride) {
        bool uni = true;
#pragma unroll
        for (int u = 0; u < kPatU; ++u) uni &= q[u] < 0 || (q[u] & 31) == pid;
        if (!uni) return k0;
        int qn[kPatU];
        sell_pattern_ids(patlist, npatc, k0 + kPatU * stride, stride, qn);
#if PEPP_PAT_PREFETCH
        // the rows of x of the group PEPP_PAT_PREFETCH steps ahead: the band
        // of chunks the whole grid works on then touches them first (DRAM),
        // so pull them into L2 now
        {
            int qp[kPatU];
            if (PEPP_PAT_PREFETCH == 1) {
#pragma unroll
                for (int u = 0; u < kPatU; ++u) qp[u] = qn[u];
            } else {
                sell_pattern_ids(patlist, npatc, k0 + PEPP_PAT_PREFETCH * kPatU * stride, stride, qp);
            }
#pragma unroll
            for (int u = 0; u < kPatU; ++u)
                if (qp[u] >= 0) asm volatile("prefetch.global.L2 [%0];" ::"l"(x + (qp[u] >> 5) * 32 + lane));
        }
#endif
        // at most ~20 gathers in flight per lane: long patterns take the
        // group in sub-groups of H chunks (keeps the kernel at 48 registers)
        constexpr int H = N * kPatU > PEPP_PAT_INFLIGHT ? (PEPP_PAT_INFLIGHT / N > 0 ? PEPP_PAT_INFLIGHT / N : 1) : kPatU;
#pragma unroll
        for (int u0 = 0; u0 < kPatU; u0 += H) {
            T xv[H][N];
#pragma unroll
            for (int u = 0; u < H; ++u) {
                const int qq = u0 + u < kPatU ? q[u0 + u] : -1;
                const int r = (qq >> 5) * 32 + lane;
#pragma unroll
                for (int j = 0; j < N; ++j) xv[u][j] = qq >= 0 ? ld_x(x, r + o[j]) : T(0);
            }
#pragma unroll
            for (int u = 0; u < H; ++u) {
                const int qq = u0 + u < kPatU ? q[u0 + u] : -1;
                T acc = T(0);
#pragma unroll
                for (int j = 0; j < N; ++j) acc = fma(v[j], xv[u][j], acc);   // slot order = the row's CSR order
                if (qq >= 0) y[(qq >> 5) * 32 + lane] = acc;
            }
        }
#pragma unroll
        for (int u = 0; u < kPatU; ++u) q[u] = qn[u];
    }
    return k0;
}

template <typename T>
__device__ __forceinline__ T sell_pattern_chunk(const SellPatterns<T>& pt, int pid, int row0,
                                                const T* __restrict__ x) {
    switch (pt.len[pid]) {
    case 1: return sell_pattern_slots<1, T>(pt, pid, row0, x);
    case 2: return sell_pattern_slots<2, T>(pt, pid, row0, x);
    case 3: return sell_pattern_slots<3, T>(pt, pid, row0, x);
    case 4: return sell_pattern_slots<4, T>(pt, pid, row0, x);
    case 5: return sell_pattern_slots<5, T>(pt, pid, row0, x);
    case 6: return sell_pattern_slots<6, T>(pt, pid, row0, x);
    case 7: return sell_pattern_slots<7, T>(pt, pid, row0, x);
    case 8: return sell_pattern_slots<8, T>(pt, pid, row0, x);
    default: break;
    }
    if constexpr (kSellMaxPatternLen > 8) {
        switch (pt.len[pid]) {
        case 9: return sell_pattern_slots<9, T>(pt, pid, row0, x);
        case 10: return sell_pattern_slots<10, T>(pt, pid, row0, x);
        case 11: return sell_pattern_slots<11, T>(pt, pid, row0, x);
        case 12: return sell_pattern_slots<12, T>(pt, pid, row0, x);
        case 13: return sell_pattern_slots<13, T>(pt, pid, row0, x);
        case 14: return sell_pattern_slots<14, T>(pt, pid, row0, x);
        case 15: return sell_pattern_slots<15, T>(pt, pid, row0, x);
        case 16: return sell_pattern_slots<16, T>(pt, pid, row0, x);
        default: break;
        }
    }
    return T(0);
}

// Stencil list (σ = 1 plans whose stencil chunks keep their values, i.e. not
// pattern chunks): the unmasked stencil chunks of up to 8 slots, as entries
// {chunk | pattern id << 26, chunk_ptr / 32} grouped by their offset pattern;
// the distinct offset sets (<= 32) travel in the kernel's parameter space.
// A warp walks its entries U at a time with the pattern's offsets held in
// registers — no chunk descriptor, no per-lane offset load, no masks: per
// chunk only the value stream, the x gathers and the y store. The other
// chunks go through sell_kernel over the plan's genlist.
constexpr int kSellMaxStencils = 32;
constexpr int kSellMaxStencilLen = 16;   // slots of a stencil-list chunk (9-point / banded b = 4 fit)
#ifndef PEPP_SLIST_U_F64
#define PEPP_SLIST_U_F64 12   // measured (tools/gpu_u64.sh, 2 repeats): U = 6 / 8 / 12 / 16 -> 565.6 / 573.4 / 562.5 / 567.6 us on config 4; tools/gpu_u_sweep2.sh: U = 10 / 12 / 14 -> 565.5-566.5 / 560.0-570.2 / 564.9 us
#endif
#ifndef PEPP_SLIST_U_F32
#define PEPP_SLIST_U_F32 5   // U = 2 / 4 / 8 -> 373 / 360 / 459 us, general walk 421; tools/gpu_u_sweep2.sh (2 repeats): U = 3 / 4 / 5 / 6 -> 360.5 / 350.2-350.4 / 340.6-340.7 / 345.7 (one 589 outlier) us
#endif
#ifndef PEPP_SLIST_U_F64_LONG
#define PEPP_SLIST_U_F64_LONG 10   // fp64, offset sets of 9-16 slots (banded / 9-point); tools/gpu_ulong.sh (2 repeats, banded b = 4 at 10^8 rows): U = 6 / 8 / 10 / 12 -> 1404 / 1333-1334 / 1318.6 / 1325-1329 us
#endif
template <typename T, int NMAX = 8>
constexpr int sell_slist_u() {
    return std::is_same<T, float>::value ? PEPP_SLIST_U_F32 : (NMAX > 8 ? PEPP_SLIST_U_F64_LONG : PEPP_SLIST_U_F64);
}
struct SellStencils {
    int len[kSellMaxStencils];
    int off[kSellMaxStencils][kSellMaxStencilLen];
};

template <int U>
__device__ __forceinline__ void sell_slist_ids(const int2* __restrict__ list, int n, int k0, int stride,
                                               int2 (&q)[U]) {
#pragma unroll
    for (int u = 0; u < U; ++u) {
        const int kk = k0 + u * stride;
        q[u] = kk < n ? __ldg(list + kk) : make_int2(-1, 0);
    }
}

template <int U, int N, typename T>
__device__ __forceinline__ void sell_slist_chunks(const int (&o)[N], const int2 (&q)[U], int lane,
                                                  const T* __restrict__ val, const T* __restrict__ x,
                                                  T* __restrict__ y, uint64_t pol) {
    // at most ~40 values + gathers in flight per lane: long stencils take the
    // group in sub-groups of H chunks
    constexpr int H = U * N > 40 ? (40 / N > 0 ? 40 / N : 1) : U;
#pragma unroll
    for (int u0 = 0; u0 < U; u0 += H) {
        T v[H][N], xv[H][N];
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int u = u0 + h < U ? u0 + h : U - 1;
            const bool ok = u0 + h < U && q[u].x >= 0;
            const int64_t base = (int64_t)q[u].y * 32 + lane;
#pragma unroll
            for (int j = 0; j < N; ++j) v[h][j] = ok ? ld_stream_v(val + base + (int64_t)j * 32, pol) : T(0);
        }
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int u = u0 + h < U ? u0 + h : U - 1;
            const bool ok = u0 + h < U && q[u].x >= 0;
            const int r = (q[u].x & ((1 << 26) - 1)) * 32 + lane;
#pragma unroll
            for (int j = 0; j < N; ++j) xv[h][j] = ok ? ld_x(x, r + o[j]) : T(0);
        }
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int u = u0 + h < U ? u0 + h : U - 1;
            const bool ok = u0 + h < U && q[u].x >= 0;
            T acc = T(0);
#pragma unroll
            for (int j = 0; j < N; ++j) acc = fma(v[h][j], xv[h][j], acc);   // slot order = the row's CSR order
            if (ok) y[(q[u].x & ((1 << 26) - 1)) * 32 + lane] = acc;
        }
    }
}

// a run of groups whose entries all have pattern `pid` (N slots); returns
// the list index of the first group that does not (q then holds it)
template <int U, int N, typename T>
__device__ __forceinline__ int sell_slist_run(const SellStencils& st, int pid, const int2* __restrict__ list, int n,
                                              int k0, int stride, int2 (&q)[U], int lane, const T* __restrict__ val,
                                              const T* __restrict__ x, T* __restrict__ y, uint64_t pol) {
    int o[N];
#pragma unroll
    for (int j = 0; j < N; ++j) o[j] = st.off[pid][j];
    for (; k0 < n; k0 += U * stride) {
        bool uni = true;
#pragma unroll
        for (int u = 0; u < U; ++u) uni &= q[u].x < 0 || (q[u].x >> 26) == pid;
        if (!uni) return k0;
        int2 qn[U];
        sell_slist_ids<U>(list, n, k0 + U * stride, stride, qn);
        sell_slist_chunks<U, N, T>(o, q, lane, val, x, y, pol);
#pragma unroll
        for (int u = 0; u < U; ++u) q[u] = qn[u];
    }
    return k0;
}

template <int U, int N, typename T>
__device__ __forceinline__ void sell_slist_one(const SellStencils& st, int2 e, int lane, const T* __restrict__ val,
                                               const T* __restrict__ x, T* __restrict__ y, uint64_t pol) {
    int o[N];
    const int pid = e.x >> 26;
#pragma unroll
    for (int j = 0; j < N; ++j) o[j] = st.off[pid][j];
    int2 q[U];
    q[0] = e;
#pragma unroll
    for (int u = 1; u < U; ++u) q[u] = make_int2(-1, 0);
    sell_slist_chunks<U, N, T>(o, q, lane, val, x, y, pol);
}

// NMAX: the longest offset set the plan's table holds (8 or 16): plans with
// short stencils get the instance whose registers are sized for them
template <int U, int NMAX, typename T>
__device__ __forceinline__ int sell_slist_dispatch_run(int len, const SellStencils& st, int pid,
                                                       const int2* __restrict__ list, int n, int k0, int stride,
                                                       int2 (&e)[U], int lane, const T* __restrict__ val,
                                                       const T* __restrict__ x, T* __restrict__ y, uint64_t pol) {
#define PEPP_SLR(N) case N: return sell_slist_run<U, N, T>(st, pid, list, n, k0, stride, e, lane, val, x, y, pol);
    switch (len) {
    PEPP_SLR(1) PEPP_SLR(2) PEPP_SLR(3) PEPP_SLR(4) PEPP_SLR(5) PEPP_SLR(6) PEPP_SLR(7)
    default: break;
    }
    if constexpr (NMAX > 8) {
        switch (len) {
        PEPP_SLR(8) PEPP_SLR(9) PEPP_SLR(10) PEPP_SLR(11) PEPP_SLR(12) PEPP_SLR(13) PEPP_SLR(14) PEPP_SLR(15)
        default: break;
        }
        return sell_slist_run<U, 16, T>(st, pid, list, n, k0, stride, e, lane, val, x, y, pol);
    }
    return sell_slist_run<U, 8, T>(st, pid, list, n, k0, stride, e, lane, val, x, y, pol);
#undef PEPP_SLR
}

template <int U, int NMAX, typename T>
__device__ __forceinline__ void sell_slist_dispatch_one(int len, const SellStencils& st, int2 e, int lane,
                                                        const T* __restrict__ val, const T* __restrict__ x,
                                                        T* __restrict__ y, uint64_t pol) {
#define PEPP_SLO(N) case N: sell_slist_one<U, N, T>(st, e, lane, val, x, y, pol); return;
    switch (len) {
    PEPP_SLO(1) PEPP_SLO(2) PEPP_SLO(3) PEPP_SLO(4) PEPP_SLO(5) PEPP_SLO(6) PEPP_SLO(7)
    default: break;
    }
    if constexpr (NMAX > 8) {
        switch (len) {
        PEPP_SLO(8) PEPP_SLO(9) PEPP_SLO(10) PEPP_SLO(11) PEPP_SLO(12) PEPP_SLO(13) PEPP_SLO(14) PEPP_SLO(15)
        default: break;
        }
        sell_slist_one<U, 16, T>(st, e, lane, val, x, y, pol);
        return;
    }
    sell_slist_one<U, 8, T>(st, e, lane, val, x, y, pol);
#undef PEPP_SLO
}

#ifndef PEPP_SLIST_MINB_F32
#define PEPP_SLIST_MINB_F32 1   // experiments: minimum resident blocks per SM for the fp32 list kernel
#endif
template <int BLOCK, int U, int NMAX, typename T>
__global__ void __launch_bounds__(BLOCK, std::is_same<T, float>::value ? PEPP_SLIST_MINB_F32 : 1) sell_slist_kernel(const int2* __restrict__ list, int n,
                                                           const __grid_constant__ SellStencils st,
                                                           const T* __restrict__ val, const T* __restrict__ x,
                                                           T* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int warp = (blockIdx.x * BLOCK + threadIdx.x) >> 5;
    const int nwarps = (gridDim.x * BLOCK) >> 5;
    const uint64_t pol = evict_first_policy();
    int2 e[U];
    int k0 = warp;
    sell_slist_ids<U>(list, n, k0, nwarps, e);
    while (k0 < n) {
        const int pid = e[0].x >> 26;
        k0 = sell_slist_dispatch_run<U, NMAX, T>(st.len[pid], st, pid, list, n, k0, nwarps, e, lane, val, x, y, pol);
        if (k0 >= n) break;
        for (int u = 0; u < U; ++u)   // a group that straddles two offset sets
            if (e[u].x >= 0) sell_slist_dispatch_one<U, NMAX, T>(st.len[e[u].x >> 26], st, e[u], lane, val, x, y, pol);
        k0 += U * nwarps;
        sell_slist_ids<U>(list, n, k0, nwarps, e);
    }
}

struct NoPatterns {};
template <bool PAT, typename T>
using SellPatternArg = std::conditional_t<PAT, SellPatterns<T>, NoPatterns>;

// Phase B of sell_kernel (and the grid-edge walk inside the tile kernel):
// warp `warp` of `nwarps` walks its chunks (σ = 1: i = warp, + nwarps, ...
// over `genlist` when PAT, else over all chunks; σ > 1: the plan-time range
// wstart[warp] .. wstart[warp + 1] of the transposed window order).
template <bool SORTED, bool PAT, typename T>
__device__ __forceinline__ void sell_walk(int nrows, int nchunks, const int64_t* __restrict__ chunk_ptr,
                                          const int* __restrict__ chunk_len, const int* __restrict__ rowlen,
                                          const int* __restrict__ perm, const int* __restrict__ col,
                                          const int16_t* __restrict__ col16, const int* __restrict__ soff,
                                          const SellPatternArg<PAT, T>& pt, const T* __restrict__ val,
                                          const T* __restrict__ x, T* __restrict__ y, int cpw,
                                          const int* __restrict__ wstart, const int* __restrict__ genlist, int warp,
                                          int nwarps, int lane, uint64_t pol) {
    const int nfull = SORTED ? (nchunks / cpw) * cpw : 0;
    const int nwin = SORTED ? nchunks / cpw : 1;
    auto chunk_of = [&](int i) -> int {
        if (!SORTED) return PAT ? __ldg(genlist + i) : i;
        return i < nfull ? (i % nwin) * cpw + i / nwin : i;
    };
    // Two-deep software pipelining over the warp's chunks (latency-bound
    // kernel): while chunk i computes, chunk i+1's dependent per-lane loads
    // (row length if masked, original row if sorted, the stencil offsets —
    // lane j loads slot j's offset once, broadcast later with shuffles) and
    // chunk i+2's descriptor (length/flags, slot pointer) are in flight.
    struct Desc { int d; int64_t cp; };
    struct Lane { int len; int orow; int offl; };
    int i = warp, end = nchunks, step = nwarps;
    if (SORTED) { i = __ldg(wstart + warp); end = __ldg(wstart + warp + 1); step = 1; }
    auto desc = [&](int i) -> Desc {
        Desc q{0, 0};
        if (i < end) { const int c = chunk_of(i); q.d = __ldg(chunk_len + c); q.cp = __ldg(chunk_ptr + c); }
        return q;
    };
    auto lanes = [&](int i, const Desc& q) -> Lane {
        Lane l{0, 0, 0};
        if (i >= end) return l;
        const int c = chunk_of(i);
        const int r = c * 32 + lane;
        l.len = !(q.d & kSellMasked) ? (q.d & kSellLenMask) : (r < nrows ? __ldg(rowlen + r) : 0);
        l.orow = (SORTED && r < nrows) ? __ldg(perm + r) : r;
        if ((q.d & kSellStencil) && lane < (q.d & kSellLenMask)) l.offl = __ldg(soff + (q.cp >> 5) + lane);
        return l;
    };
    Desc q0 = desc(i), q1 = desc(i + step);
    Lane l0 = lanes(i, q0);
    for (; i < end; i += step) {
        const Desc q2 = desc(i + 2 * step);
        const Lane l1 = lanes(i + step, q1);
        if constexpr ((sell_pairs<T>() && !SORTED && !PAT) || (PEPP_SELL_PAIR_SORTED && SORTED && !PAT)) {
            // chunks i and i+1 both unmasked stencil chunks of one length <= 8:
            // both at once, then the pipeline moves two chunks on (σ > 1: the
            // transposed window order puts chunks of equal length next to each
            // other, any index format)
            const int pl = q0.d & kSellLenMask;
            const bool fmt_ok = (q0.d & kSellStencil) || PEPP_SELL_PAIR_ALL || SORTED;
            if (q1.d == q0.d && fmt_ok && !(q0.d & kSellMasked) && pl >= 1 && pl <= 8 && i + step < end) {
                const int ra = l0.orow, rb = l1.orow;
                T a = T(0), b = T(0);
                if (q0.d & kSellStencil)
                    sell_pair_len<kIdxStencil, T>(pl, val, col, col16, x, l0.offl, ra, q0.cp + lane, l1.offl, rb, q1.cp + lane, a, b, pol);
                else if (q0.d & kSellCol16)
                    sell_pair_len<kIdx16, T>(pl, val, col, col16, x, 0, ra, q0.cp + lane, 0, rb, q1.cp + lane, a, b, pol);
                else
                    sell_pair_len<kIdx32, T>(pl, val, col, col16, x, 0, ra, q0.cp + lane, 0, rb, q1.cp + lane, a, b, pol);
                y[ra] = a;   // unmasked chunks: all 32 rows exist
                y[rb] = b;
                const Desc q3 = desc(i + 3 * step);
                l0 = lanes(i + 2 * step, q2);
                q0 = q2; q1 = q3;
                i += step;   // + the loop's step
                continue;
            }
        }
        const int c = chunk_of(i);
        const int64_t base = q0.cp + lane;
        const int clen = q0.d & kSellLenMask;
        T acc;
        bool pat_chunk = false;
        if constexpr (PAT) {
            pat_chunk = (q0.d & kSellPattern) != 0;
            if (pat_chunk) acc = sell_pattern_chunk<T>(pt, (int)q0.cp, l0.orow, x);   // cp holds the pattern id
        }
        if (pat_chunk) {
        } else if (q0.d & kSellStencil) acc = sell_chunk<kIdxStencil, T>(val, col, col16, l0.offl, l0.orow, x, base, clen, l0.len, pol);
        else if (q0.d & kSellCol16) acc = sell_chunk<kIdx16, T>(val, col, col16, 0, l0.orow, x, base, clen, l0.len, pol);
        else acc = sell_chunk<kIdx32, T>(val, col, col16, 0, l0.orow, x, base, clen, l0.len, pol);
        if (c * 32 + lane < nrows) y[l0.orow] = acc;
        q0 = q1; q1 = q2; l0 = l1;
    }
}

// PAT: the plan has pattern chunks (phase A + genlist); PAT = false compiles
// the general kernel without them (no extra registers, no 3 KB parameter).
#ifndef PEPP_PAT_MINB
#define PEPP_PAT_MINB 2   // minimum resident blocks per SM for the σ = 1 PAT (value-compressed) instance: with 16-slot patterns it would take 208 registers (1 block per SM)
#endif
template <int BLOCK, bool SORTED, bool PAT, typename T>
__global__ void __launch_bounds__(BLOCK, (PAT && !SORTED) ? PEPP_PAT_MINB : 1) sell_kernel(int nrows, int nchunks, const int64_t* __restrict__ chunk_ptr,
                                                     const int* __restrict__ chunk_len,
                                                     const int* __restrict__ rowlen,
                                                     const int* __restrict__ perm,
                                                     const int* __restrict__ col,
                                                     const int16_t* __restrict__ col16,
                                                     const int* __restrict__ soff,
                                                     const __grid_constant__ SellPatternArg<PAT, T> pt,
                                                     const T* __restrict__ val,
                                                     const T* __restrict__ x,
                                                     T* __restrict__ y,
                                                     int cpw,
                                                     const int* __restrict__ wstart,
                                                     const int* __restrict__ patlist, int npatc,
                                                     const int* __restrict__ genlist) {
    const int lane = threadIdx.x & 31;
    const int warp = (blockIdx.x * BLOCK + threadIdx.x) >> 5;
    const int nwarps = (gridDim.x * BLOCK) >> 5;
    const uint64_t pol = evict_first_policy();
    // Phase A (σ = 1 plans with pattern chunks): the pattern chunks, listed
    // as (chunk << 5 | pattern id), in a tight loop — no descriptor, no
    // per-lane loads: 1 list entry (prefetched one step ahead), the x
    // gathers, the FMAs and the y store per chunk. Phase B below then walks
    // only the other chunks (`genlist`, `nchunks` of them).
    if constexpr (!SORTED && PAT) if (npatc > 0) {
        // Runs of one pattern go through sell_pattern_run<N> (no per-chunk
        // branch on the pattern length); a group of list entries that
        // straddles two patterns (the list is sorted by id: at most one per
        // pattern change per warp) takes the one-chunk path.
        int e[kPatU];
        int k0 = warp;
        sell_pattern_ids(patlist, npatc, k0, nwarps, e);
        while (k0 < npatc) {
            const int pid = e[0] & 31;
            switch (pt.len[pid]) {
            case 1: k0 = sell_pattern_run<1, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
            case 2: k0 = sell_pattern_run<2, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
            case 3: k0 = sell_pattern_run<3, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
            case 4: k0 = sell_pattern_run<4, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
            case 5: k0 = sell_pattern_run<5, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
            case 6: k0 = sell_pattern_run<6, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
            case 7: k0 = sell_pattern_run<7, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
            case 8: k0 = sell_pattern_run<8, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
            default:
                if constexpr (kSellMaxPatternLen > 8) {
                    switch (pt.len[pid]) {
                    case 9: k0 = sell_pattern_run<9, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
                    case 10: k0 = sell_pattern_run<10, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
                    case 11: k0 = sell_pattern_run<11, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
                    case 12: k0 = sell_pattern_run<12, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
                    case 13: k0 = sell_pattern_run<13, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
                    case 14: k0 = sell_pattern_run<14, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
                    case 15: k0 = sell_pattern_run<15, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
                    default: k0 = sell_pattern_run<16, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y); break;
                    }
                } else {
                    k0 = sell_pattern_run<8, T>(pt, pid, patlist, npatc, k0, nwarps, e, lane, x, y);
                }
                break;
            }
            if (k0 >= npatc) break;
            for (int u = 0; u < kPatU; ++u) {   // the mixed group
                if (e[u] < 0) continue;
                const int r = (e[u] >> 5) * 32 + lane;
                y[r] = sell_pattern_chunk<T>(pt, e[u] & 31, r, x);
            }
            k0 += kPatU * nwarps;
            sell_pattern_ids(patlist, npatc, k0, nwarps, e);
        }
    }
    sell_walk<SORTED, PAT, T>(nrows, nchunks, chunk_ptr, chunk_len, rowlen, perm, col, col16, soff, pt, val, x, y, cpw,
                              wstart, genlist, warp, nwarps, lane, pol);
}

// =====================================================================
// Variant 1: merge-path CSR (balanced over rows + nonzeros).
// The merge of the row-end list (rp[1..nrows]) with the nonzero indices is
// cut into tiles of TILE = BLOCK*IPT items; tile start coordinates are
// found once at plan time (merge_tile_search). Per tile: stage the tile's
// row ends and the products val*x[col] in shared memory with coalesced
// loads, then each thread consumes IPT merge items sequentially. Rows that
// cross thread boundaries are joined with a deterministic block-wide
// segmented scan; rows that cross tile boundaries leave a carry that
// merge_fixup_kernel adds afterwards, in tile order (no fp atomics).
// =====================================================================
template <typename T>
struct SegPairT {
    T v;
    int f;  // 1 = a row ended inside this segment (resets the running sum)
};
template <typename T>
__device__ __forceinline__ SegPairT<T> seg_combine(SegPairT<T> a, SegPairT<T> b) {
    // a precedes b
    SegPairT<T> r;
    r.f = a.f | b.f;
    r.v = b.f ? b.v : a.v + b.v;
    return r;
}

template <int BLOCK, int IPT, typename T>
__global__ void __launch_bounds__(BLOCK) merge_spmv_kernel(int nrows, const int* __restrict__ rp,
                                                          const int* __restrict__ col,
                                                          const T* __restrict__ val,
                                                          const T* __restrict__ x,
                                                          T* __restrict__ y,
                                                          const int2* __restrict__ tile_coord,
                                                          int* __restrict__ carry_row,
                                                          T* __restrict__ carry_val) {
    using SegPair = SegPairT<T>;
    constexpr int TILE = BLOCK * IPT;
    constexpr int NW = BLOCK / 32;
    __shared__ int s_row_end[TILE];
    __shared__ T s_prod[TILE];
    __shared__ SegPair s_warp[NW];

    const int tid = threadIdx.x;
    const int tile = blockIdx.x;
    const int2 c0 = __ldg(tile_coord + tile);
    const int2 c1 = __ldg(tile_coord + tile + 1);
    const int nr = c1.x - c0.x;   // row ends in this tile
    const int nz = c1.y - c0.y;   // nonzeros in this tile

    const uint64_t pol = evict_first_policy();
    // staging, batched per thread: every thread owns IPT slots of each list
    // (nr, nz <= TILE = BLOCK*IPT); all index/value loads are issued, then all
    // x gathers, then the products are stored — no serial load chains.
    {
        int re[IPT], ci[IPT];
        T v[IPT], xv[IPT];
#pragma unroll
        for (int u = 0; u < IPT; ++u) {
            const int i = tid + u * BLOCK;
            re[u] = i < nr ? __ldg(rp + c0.x + 1 + i) : 0;
            ci[u] = i < nz ? ld_stream_i(col + c0.y + i, pol) : 0;
            v[u] = i < nz ? ld_stream_v(val + c0.y + i, pol) : T(0);
        }
#pragma unroll
        for (int u = 0; u < IPT; ++u) xv[u] = (tid + u * BLOCK < nz) ? ld_x_ordered(x, ci[u]) : T(0);
#pragma unroll
        for (int u = 0; u < IPT; ++u) {
            const int i = tid + u * BLOCK;
            if (i < nr) s_row_end[i] = re[u];
            if (i < nz) s_prod[i] = v[u] * xv[u];
        }
    }
    __syncthreads();

    // this thread's start on the tile-local merge path
    const int total = nr + nz;
    const int d = min(tid * IPT, total);
    int lo = max(0, d - nz), hi = min(d, nr);
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (s_row_end[mid] <= c0.y + d - mid - 1) lo = mid + 1;
        else hi = mid;
    }
    int ri = lo, ki = d - lo;
    const int dend = min(d + IPT, total);

    T acc = T(0), head_val = T(0);
    int head_row = -1;
#pragma unroll
    for (int it = 0; it < IPT; ++it) {
        if (d + it < dend) {
            const int re = ri < nr ? s_row_end[ri] : 0x7fffffff;
            if (c0.y + ki < re) {                   // consume a nonzero
                acc += s_prod[ki];
                ++ki;
            } else {                                // row ri ends here
                if (head_row < 0) { head_row = ri; head_val = acc; }
                else y[c0.x + ri] = acc;
                acc = T(0);
                ++ri;
            }
        }
    }

    // block-wide inclusive segmented scan of (acc, ended-a-row)
    SegPair me{acc, head_row >= 0 ? 1 : 0};
    SegPair inc = me;
    const int lane = tid & 31, wid = tid >> 5;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        SegPair o;
        o.v = __shfl_up_sync(0xffffffffu, inc.v, off);
        o.f = __shfl_up_sync(0xffffffffu, inc.f, off);
        if (lane >= off) inc = seg_combine(o, inc);
    }
    if (lane == 31) s_warp[wid] = inc;
    __syncthreads();
    SegPair wpre{T(0), 0};
    for (int w = 0; w < wid; ++w) wpre = w == 0 ? s_warp[0] : seg_combine(wpre, s_warp[w]);
    // exclusive prefix for this thread = (warp prefix) ⊕ (inclusive of lane-1)
    SegPair prev;
    prev.v = __shfl_up_sync(0xffffffffu, inc.v, 1);
    prev.f = __shfl_up_sync(0xffffffffu, inc.f, 1);
    SegPair excl;
    if (lane == 0) excl = wpre;
    else excl = (wid == 0) ? prev : seg_combine(wpre, prev);
    if (wid == 0 && lane == 0) excl = SegPair{T(0), 0};

    if (head_row >= 0) y[c0.x + head_row] = excl.v + head_val;

    if (tid == BLOCK - 1) {
        const SegPair all = (wid == 0) ? inc : seg_combine(wpre, inc);
        carry_row[tile] = c1.x;            // the row left open at the end of the tile
        carry_val[tile] = all.v;
    }
}

// Warp-granular merge-path: the same decomposition with tiles of 32*IPT
// merge items owned by ONE warp (row ends + products staged in that warp's
// slice of shared memory, warp-only segmented scan): no block barriers, so
// every warp streams independently (latency hiding by warp count).
template <int IPT, int WARPS, typename T>
__global__ void __launch_bounds__(WARPS * 32) merge_warp_kernel(int nrows, int ntiles, const int* __restrict__ rp,
                                                               const int* __restrict__ col,
                                                               const T* __restrict__ val,
                                                               const T* __restrict__ x,
                                                               T* __restrict__ y,
                                                               const int2* __restrict__ tile_coord,
                                                               int* __restrict__ carry_row,
                                                               T* __restrict__ carry_val) {
    using SegPair = SegPairT<T>;
    constexpr int TILE = 32 * IPT;
    __shared__ int s_row_end_all[WARPS][TILE];
    __shared__ T s_prod_all[WARPS][TILE];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int tile = blockIdx.x * WARPS + w;
    if (tile >= ntiles) return;
    int* s_row_end = s_row_end_all[w];
    T* s_prod = s_prod_all[w];
    const uint64_t pol = evict_first_policy();
    const int2 c0 = __ldg(tile_coord + tile);
    const int2 c1 = __ldg(tile_coord + tile + 1);
    const int nr = c1.x - c0.x, nz = c1.y - c0.y;
    {
        int re[IPT], ci[IPT];
        T v[IPT], xv[IPT];
#pragma unroll
        for (int u = 0; u < IPT; ++u) {
            const int i = lane + u * 32;
            re[u] = i < nr ? __ldg(rp + c0.x + 1 + i) : 0;
            ci[u] = i < nz ? ld_stream_i(col + c0.y + i, pol) : 0;
            v[u] = i < nz ? ld_stream_v(val + c0.y + i, pol) : T(0);
        }
#pragma unroll
        for (int u = 0; u < IPT; ++u) xv[u] = (lane + u * 32 < nz) ? ld_x_ordered(x, ci[u]) : T(0);
#pragma unroll
        for (int u = 0; u < IPT; ++u) {
            const int i = lane + u * 32;
            if (i < nr) s_row_end[i] = re[u];
            if (i < nz) s_prod[i] = v[u] * xv[u];
        }
    }
    __syncwarp();
    const int total = nr + nz;
    const int d = min(lane * IPT, total);
    int lo = max(0, d - nz), hi = min(d, nr);
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (s_row_end[mid] <= c0.y + d - mid - 1) lo = mid + 1;
        else hi = mid;
    }
    int ri = lo, kabs = c0.y + d - lo;
    const int dend = min(d + IPT, total);
    int re = ri < nr ? s_row_end[ri] : 0x7fffffff;
    T acc = T(0), head_val = T(0);
    int head_row = -1;
#pragma unroll
    for (int it = 0; it < IPT; ++it) {
        if (d + it < dend) {
            if (kabs < re) {
                acc += s_prod[kabs - c0.y];
                ++kabs;
            } else {
                if (head_row < 0) { head_row = ri; head_val = acc; }
                else y[c0.x + ri] = acc;
                acc = T(0);
                ++ri;
                re = ri < nr ? s_row_end[ri] : 0x7fffffff;
            }
        }
    }
    // warp inclusive segmented scan of (acc, ended-a-row)
    SegPair inc{acc, head_row >= 0 ? 1 : 0};
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        SegPair o;
        o.v = __shfl_up_sync(0xffffffffu, inc.v, off);
        o.f = __shfl_up_sync(0xffffffffu, inc.f, off);
        if (lane >= off) inc = seg_combine(o, inc);
    }
    T excl = __shfl_up_sync(0xffffffffu, inc.v, 1);
    if (lane == 0) excl = T(0);
    if (head_row >= 0) y[c0.x + head_row] = excl + head_val;
    if (lane == 31) {
        carry_row[tile] = c1.x;
        carry_val[tile] = inc.v;
    }
}

// Carry fix-up. Tile t leaves carry_val[t] for row carry_row[t] (the row
// open at its end); a run of consecutive tiles carrying into one row is
// summed in tile order and added to y[row] once (deterministic, no fp
// atomics). Runs are fixed by the matrix structure, so the plan lists the
// long ones (>= kLongRun tiles, rows spanning many tiles): those go to
// merge_fixup_long_kernel (one warp per run, lane-strided + fixed shuffle
// tree); merge_fixup_kernel (one thread per tile) handles the short ones.
constexpr int kLongRun = 32;

template <typename T>
__global__ void merge_fixup_kernel(int ntiles, int nrows, const int* __restrict__ carry_row,
                                   const T* __restrict__ carry_val, T* __restrict__ y) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= ntiles) return;
    const int row = carry_row[t];
    if (row >= nrows) return;
    if (t > 0 && carry_row[t - 1] == row) return;
    T s = carry_val[t];
    int u = t + 1;
    for (; u < ntiles && u - t < kLongRun && carry_row[u] == row; ++u) s += carry_val[u];
    if (u - t >= kLongRun) return;   // a long run: merge_fixup_long_kernel adds it
    y[row] = s + y[row];
}

// runs[i] = (first tile, number of tiles, row)
template <typename T>
__global__ void merge_fixup_long_kernel(int nruns, const int4* __restrict__ runs, const T* __restrict__ carry_val,
                                        T* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int i = (int)((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    if (i >= nruns) return;
    const int4 r = runs[i];
    T s = T(0);
    for (int u = lane; u < r.y; u += 32) s += carry_val[r.x + u];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) y[r.z] = s + y[r.z];
}

// Plan time: tile start coordinates on the global merge path.
__global__ void merge_tile_search_kernel(int nrows, int64_t nnz, const int* __restrict__ rp, int tile_items,
                                         int ntiles, int2* __restrict__ tile_coord) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t > ntiles) return;
    const int base = rp[0];
    const int64_t total = (int64_t)nrows + nnz;
    const int64_t d = min((int64_t)t * tile_items, total);
    int64_t lo = max((int64_t)0, d - nnz), hi = min(d, (int64_t)nrows);
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if ((int64_t)rp[mid + 1] - base <= d - mid - 1) lo = mid + 1;
        else hi = mid;
    }
    tile_coord[t] = make_int2((int)lo, (int)(base + (d - lo)));
}

// =====================================================================
// Variant 3: CSR-stream with a TMA bulk-copy pipeline (B200-native).
// The matrix is cut at plan time into work items of <= NB nonzeros and
// <= RMAX rows (rows longer than NB become "pieces" of NB nonzeros). A
// persistent CTA owns items b, b+G, b+2G, ...; one thread streams each
// item's row_ptr slice, columns and values into a STAGES-deep shared-memory
// ring with cp.async.bulk (completion counted on an mbarrier per stage),
// so STAGES-1 items are in flight while the CTA computes the current one:
//   phase 1 (balanced over nonzeros): sval[k] <- val[k] * x[col[k]]
//   phase 2 (per row): rows of <= VEC entries: one thread sums the row's
//           products sequentially from +0.0 — the oracle's exact arithmetic
//           (product rounded, then each sum rounded, ascending k), so those
//           rows are bit-identical to the definition; rows of VEC..NB
//           entries: one warp per row, lane-strided + shuffle tree; rows
//           longer than NB: NB-sized pieces, each a block-wide sum written to
//           a carry slot, combined in piece order by csr_stream_fixup_kernel.
// =====================================================================
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    uint32_t done;
    do {
        asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
                     : "=r"(done) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    } while (!done);
}
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void tma_load_1d_nohint(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void tma_store_1d(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// =====================================================================
// SELL tiles (B200-native): runs of consecutive stencil chunks of one
// offset set. A stencil chunk's 32 rows share their column offsets o_j, so
// y[r] = sum_j v_j(r) x[r + o_j]; for a run of chunks starting at row r0
// the x elements needed form, per cluster of nearby offsets (gap <= 64),
// one contiguous range [r0 + lo, r0 + nr - 1 + hi], and the chunks' values
// (slot-major per chunk, chunks consecutive in the SELL value array) one
// contiguous block. A producer warp copies each range (rounded out to 16 B:
// r0 is a multiple of 32, so the rounding is a per-set constant) and, when
// the values are streamed (VALS), the value block into a shared-memory
// stage with cp.async.bulk, completion counted on the stage's mbarrier,
// S stages deep; consumer warps compute the tile's rows from shared memory
// — per row the same FMAs in the same slot order as the register paths
// (sell_pattern_slots / sell_slist_chunks: bit-identical) — and store y.
// !VALS: pattern chunks (value compression, the values are kernel
// parameters; only x is read and y written). x elements are read once
// from DRAM (a 5-point stencil's three ranges meet again in L2 as the grid's
// front advances: ±n grid rows are ~64 KB apart), and nothing goes through
// the L1 gather path that held the register form at ~0.6 of the copy peak
// (one 32-B sector request per SM cycle: ~26 sectors per chunk). Grid
// stencils' pattern tiles come as multi-line tiles (PatTiles.D: K lines of a
// column, each x line copied once). The chunks outside the tiles (grid
// edges) are walked by the CTA's last warps with the general SELL walk.
// One persistent CTA per SM: warp 0 producer, warps 1-8 consumers, then
// the walkers (DESIGN §6 "SELL tiles" has the measured design steps).
// =====================================================================
constexpr int kTileMaxSets = 32, kTileMaxLen = 16;
struct PatTiles {
    int len[kTileMaxSets];                       // slots of set q
    int ncl[kTileMaxSets];                       // offset clusters of set q
    int clo[kTileMaxSets][kTileMaxLen];          // cluster c: first x element, relative to r0 (16-B aligned)
    int cext[kTileMaxSets][kTileMaxLen];         // elements copied = round16(nr + cext)
    int cdst[kTileMaxSets][kTileMaxLen];         // cluster c's element offset within a stage
    int sidx[kTileMaxSets][kTileMaxLen];         // slot j: stage element of the tile's row 0
    // multi-line tiles (!VALS; tile entry .z = K > 0): the set's offsets are
    // a_j·D + b_j with a_j in [amin, amax] (a grid stencil, D = the line
    // stride); a tile is K lines of nr rows, r0 + l·D (l < K), and loads the
    // K + W lines (W = amax - amin) x[r0 + lbase + m·D, + round16(nr + lext))
    // once each into stage line m (stride lws) — x crosses L2 -> SM
    // (K + W) / K times instead of once per cluster per line
    int D[kTileMaxSets], W[kTileMaxSets], lbase[kTileMaxSets], lext[kTileMaxSets], lws[kTileMaxSets];
    int msidx[kTileMaxSets][kTileMaxLen];        // slot j: stage element of line 0's row 0
};

#ifndef PEPP_PTILE_U
#define PEPP_PTILE_U 4   // rows per consumer thread per step (independent FMA chains, all loads first)
#endif
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// Consumer thread c of NC: rows c, c + NC, ... of the tile, U at a time
// (all shared-memory loads of the U rows first), written straight to y.
// VALS: slot j of row i is sv[(i / 32) * 32N + 32 j + i % 32].
#ifndef PEPP_TILE_CHECKS
#define PEPP_TILE_CHECKS 0   // 1: bounds traps in sell_tile_kernel (debug builds, tools/r2/gpu_tile_checks.sh)
#endif
template <int NC, int N, bool VALS, typename T>
__device__ __forceinline__ void tile_rows(const SellPatterns<T>& pt, const int* sidx, int q, const T* sx,
                                          const T* sv, T* __restrict__ y, int nr, int c, int xspan) {
    constexpr int U = !VALS ? (N <= 8 ? PEPP_PTILE_U : 2) : (N <= 4 ? 4 : N <= 8 ? 2 : 1);
    int b[N];
    T w[N];
#pragma unroll
    for (int j = 0; j < N; ++j) { b[j] = sidx[j]; w[j] = VALS ? T(0) : pt.val[q][j]; }
#if PEPP_TILE_CHECKS
    for (int j = 0; j < N; ++j)
        if (b[j] < 0 || b[j] + nr > xspan) __trap();   // every slot's reads inside the stage's x part
#else
    (void)xspan;
#endif
    for (int i0 = c; i0 < nr; i0 += NC * U) {
        T xv[U][N], vv[VALS ? U : 1][N];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int i = i0 + u * NC < nr ? i0 + u * NC : i0;
#pragma unroll
            for (int j = 0; j < N; ++j) xv[u][j] = sx[b[j] + i];
            if constexpr (VALS) {
                const T* v = sv + (i >> 5) * (32 * N) + (i & 31);
#pragma unroll
                for (int j = 0; j < N; ++j) vv[u][j] = v[32 * j];
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            T acc = T(0);
#pragma unroll
            for (int j = 0; j < N; ++j) acc = fma(VALS ? vv[u][j] : w[j], xv[u][j], acc);   // slot order = CSR order
            if (i0 + u * NC < nr) y[i0 + u * NC] = acc;
        }
    }
}

// tiles[t] = {first chunk, chunks << 5 | set id, value block / 32 (VALS), 0};
// persistent CTAs walk t = blockIdx.x, + gridDim.x, ... (the grid's front
// advances through the rows together, so the ranges of neighbouring tiles
// meet in L2). Warp-specialized: warp 0 (one lane) is the producer — it
// waits until stage s is released (empty[s]), writes the tile's list entry
// to the stage and issues its bulk copies (completion on full[s]); the list
// entry of its next tile is loaded one tile ahead. The other BLOCK/32 - 1
// warps consume: wait full[s], read the entry, compute their rows, store y
// with coalesced st.global, release the stage (one arrive per warp). No
// CTA-wide barrier in the loop, so the producer keeps S stages in flight
// while the consumers work (a CTA-barrier form with a bulk store of y
// measured 270-600 µs on config 4: the barriers put the compute and the
// issue of every tile on one serial path).
// Shared memory: S x stage (x ranges; VALS: then the value block at
// vstage) | S full | S empty | S entries.
// The chunks outside the tiles (grid edges: `genlist`), walked by the tile
// kernel's last NWK warps with the general SELL walk (sell_walk) while the
// producer / consumers run the tiles — beside the tiles on every SM instead
// of a second kernel on a second stream (which added 16-20 µs per call).
struct TileWalk {
    int nrows = 0, ngen = 0;
    const int64_t* chunk_ptr = nullptr;
    const int* chunk_len = nullptr;
    const int* rowlen = nullptr;
    const int* col = nullptr;
    const int16_t* col16 = nullptr;
    const int* soff = nullptr;
    const int* genlist = nullptr;
};

template <int BLOCK, int S, bool VALS, typename T, int NWK>
__global__ void __launch_bounds__(BLOCK, 1) sell_tile_kernel(const __grid_constant__ SellPatterns<T> pt,
                                                             const __grid_constant__ PatTiles tt,
                                                             const int4* __restrict__ tiles, int ntiles,
                                                             int stage_elems, int vstage,
                                                             const T* __restrict__ val, const T* __restrict__ x,
                                                             T* __restrict__ y, int64_t xlen, const TileWalk wk) {
    extern __shared__ __align__(128) unsigned char ptile_smem[];
    constexpr int A = 16 / sizeof(T);
    constexpr int NCW = BLOCK / 32 - 1 - NWK, NC = NCW * 32;
    T* sx = reinterpret_cast<T*>(ptile_smem);
    uint64_t* full = reinterpret_cast<uint64_t*>(sx + (size_t)S * stage_elems);
    uint64_t* empty = full + S;
    int4* ent = reinterpret_cast<int4*>(empty + S);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int G = gridDim.x;
    if (tid == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], NCW); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (warp > NCW) {   // the walkers: the chunks outside the tiles
        if (wk.ngen > 0)
            sell_walk<false, true, T>(wk.nrows, wk.ngen, wk.chunk_ptr, wk.chunk_len, wk.rowlen, nullptr, wk.col, wk.col16,
                                      wk.soff, pt, val, x, y, 1, nullptr, wk.genlist, blockIdx.x * NWK + (warp - NCW - 1),
                                      gridDim.x * NWK, lane, evict_first_policy());
        return;
    }
    if (warp == 0) {
        if (lane != 0) return;
        int4 e = blockIdx.x < ntiles ? __ldg(tiles + blockIdx.x) : make_int4(0, 0, 0, 0);
        for (int it = 0;; ++it) {
            const int t = blockIdx.x + it * G;
            if (t >= ntiles) break;
            const int s = it % S;
            const int4 en = t + G < ntiles ? __ldg(tiles + t + G) : make_int4(0, 0, 0, 0);
            if (it >= S) mbar_wait(&empty[s], (uint32_t)(((it / S) - 1) & 1));
            const int64_t r0 = (int64_t)e.x * 32;
            const int nr = (e.y >> 5) * 32, q = e.y & 31, nc = tt.ncl[q];
            ent[s] = e;
            if (!VALS && e.z > 0) {   // multi-line tile: K + W lines, each once
                const int nl = e.z + tt.W[q];
                const uint32_t lb = (uint32_t)(((nr + tt.lext[q] + A - 1) / A) * A) * sizeof(T);
                mbar_arrive_expect_tx(&full[s], lb * nl);
                T* dst = sx + (size_t)s * stage_elems;
                const T* src = x + r0 + tt.lbase[q];
                for (int m = 0; m < nl; ++m) {
#if PEPP_TILE_CHECKS
                    const int64_t a = r0 + tt.lbase[q] + (int64_t)m * tt.D[q];
                    if (a < 0 || a + lb / sizeof(T) > xlen || (int64_t)m * tt.lws[q] + lb / sizeof(T) > stage_elems) __trap();
#endif
                    tma_load_1d_nohint(dst + m * tt.lws[q], src + (int64_t)m * tt.D[q], lb, &full[s]);
                }
                e = en;
                continue;
            }
            uint32_t bytes = 0;
            for (int c = 0; c < nc; ++c) bytes += (uint32_t)(((nr + tt.cext[q][c] + A - 1) / A) * A) * sizeof(T);
            const uint32_t vbytes = VALS ? (uint32_t)nr * tt.len[q] * sizeof(T) : 0;
            mbar_arrive_expect_tx(&full[s], bytes + vbytes);
            T* dst = sx + (size_t)s * stage_elems;
#if PEPP_TILE_CHECKS
            // debug build (compute-sanitizer is not available on the GPU pool):
            // every copy inside x / its stage, the value block after the ranges
            for (int c = 0; c < nc; ++c) {
                const int64_t a = r0 + tt.clo[q][c], n = ((nr + tt.cext[q][c] + A - 1) / A) * A;
                if (a < 0 || a + n > xlen || tt.cdst[q][c] + n > (VALS ? vstage : stage_elems)) __trap();
            }
            if (VALS && vstage + (int64_t)nr * tt.len[q] > stage_elems) __trap();
#endif
            for (int c = 0; c < nc; ++c)
                tma_load_1d_nohint(dst + tt.cdst[q][c], x + r0 + tt.clo[q][c],
                                   (uint32_t)(((nr + tt.cext[q][c] + A - 1) / A) * A) * sizeof(T), &full[s]);
            if (VALS) tma_load_1d_nohint(dst + vstage, val + (int64_t)e.z * 32, vbytes, &full[s]);
            e = en;
        }
        return;
    }
    const int c = tid - 32;   // consumer index (warps 1 .. NCW)
    for (int it = 0;; ++it) {
        const int t = blockIdx.x + it * G;
        if (t >= ntiles) break;
        const int s = it % S;
        mbar_wait(&full[s], (uint32_t)((it / S) & 1));
        const int4 e = ent[s];
        const int nr = (e.y >> 5) * 32, q = e.y & 31;
        const T* xs = sx + (size_t)s * stage_elems;
        const T* vs = xs + vstage;
        T* yt = y + (int64_t)e.x * 32;
        if (!VALS && e.z > 0) {   // multi-line tile: line l's rows from stage line l (+ the slots' line offsets)
            for (int l = 0; l < e.z; ++l) {
                const T* xl = xs + l * tt.lws[q];
                T* yl = yt + (int64_t)l * tt.D[q];
                const int span = stage_elems - l * tt.lws[q];
#define PEPP_TM(N) case N: tile_rows<NC, N, VALS, T>(pt, tt.msidx[q], q, xl, vs, yl, nr, c, span); break;
                switch (tt.len[q]) {
                PEPP_TM(1) PEPP_TM(2) PEPP_TM(3) PEPP_TM(4) PEPP_TM(5) PEPP_TM(6) PEPP_TM(7) PEPP_TM(8)
                default:
                    if constexpr (kSellMaxPatternLen > 8) {
                        switch (tt.len[q]) {
                        PEPP_TM(9) PEPP_TM(10) PEPP_TM(11) PEPP_TM(12) PEPP_TM(13) PEPP_TM(14) PEPP_TM(15)
                        default: tile_rows<NC, 16, VALS, T>(pt, tt.msidx[q], q, xl, vs, yl, nr, c, span); break;
                        }
                    }
                    break;
                }
#undef PEPP_TM
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
            continue;
        }
#define PEPP_TR(N) case N: tile_rows<NC, N, VALS, T>(pt, tt.sidx[q], q, xs, vs, yt, nr, c, VALS ? vstage : stage_elems); break;
        switch (tt.len[q]) {
        PEPP_TR(1) PEPP_TR(2) PEPP_TR(3) PEPP_TR(4) PEPP_TR(5) PEPP_TR(6) PEPP_TR(7)
        default:
            if constexpr (VALS) {
                switch (tt.len[q]) {
                PEPP_TR(8) PEPP_TR(9) PEPP_TR(10) PEPP_TR(11) PEPP_TR(12) PEPP_TR(13) PEPP_TR(14) PEPP_TR(15)
                default: tile_rows<NC, 16, VALS, T>(pt, tt.sidx[q], q, xs, vs, yt, nr, c, VALS ? vstage : stage_elems); break;
                }
            } else if constexpr (kSellMaxPatternLen > 8) {
                switch (tt.len[q]) {
                PEPP_TR(8) PEPP_TR(9) PEPP_TR(10) PEPP_TR(11) PEPP_TR(12) PEPP_TR(13) PEPP_TR(14) PEPP_TR(15)
                default: tile_rows<NC, 16, VALS, T>(pt, tt.sidx[q], q, xs, vs, yt, nr, c, VALS ? vstage : stage_elems); break;
                }
            } else {
                tile_rows<NC, 8, VALS, T>(pt, tt.sidx[q], q, xs, vs, yt, nr, c, VALS ? vstage : stage_elems);
            }
            break;
        }
#undef PEPP_TR
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[s]);   // this warp's reads of stage s are done
    }
}

// =====================================================================
// Variant 4: column panels — random columns whose x is far larger than L2.
// With x beyond L2 (e.g. 10^8 columns = 800 MB) every random gather of the
// row-major variants is a DRAM access of its own (~50 G gathers/s). Here the
// columns are cut into panels of 2^P entries (x panel <= 64 MB, L2-resident
// while it is used) and the matrix is stored panel-major: for panel k, the
// (row, entries) pairs of the rows that have entries in it, in row order,
// each pair's entries contiguous (pcol / pval, their CSR order). One launch
// per panel, one thread per pair: the row's panel entries summed
// sequentially (product rounded by FMA, ascending column), then
// y[row] += that sum — rows are owned by one thread per panel and the
// panels run in order, so no atomics and the same bits on every call (y is
// zeroed first; row i's result is (((0 + s_0) + s_1) + ...) over the panels
// holding its entries).
// =====================================================================
// One thread per pair. (Measured alternatives, uniform 16/row: 4 pairs per
// thread with their loads interleaved 3.77 -> 4.72 ms at 3.16e7 rows and
// 15.8 -> 18.2 ms at 1e8; a warp streaming 32 pairs' entries lane-parallel
// with a segmented shuffle scan 3.86 / 17.3 ms — both slower. ncu of this
// form: DRAM at 66 % of peak, 88 % of warp samples on the dependent pair ->
// entry -> x -> y loads.)
template <typename T>
__global__ void __launch_bounds__(256) panel_kernel(int j0, int j1, const int* __restrict__ prow,
                                                    const int* __restrict__ pstart, const int* __restrict__ pcol,
                                                    const T* __restrict__ pval, const T* __restrict__ x,
                                                    T* __restrict__ y) {
    const uint64_t pol = evict_first_policy();
    for (int j = j0 + blockIdx.x * blockDim.x + threadIdx.x; j < j1; j += gridDim.x * blockDim.x) {
        const int r = __ldg(prow + j), s = __ldg(pstart + j), e = __ldg(pstart + j + 1);
        const T yv = y[r];   // issued before the entries: in flight with them, not after the FMA chain
        T acc = T(0);
        for (int k = s; k < e; ++k) acc = fma(ld_stream_v(pval + k, pol), __ldg(x + ld_stream_i(pcol + k, pol)), acc);
        y[r] = yv + acc;   // the row's panels in order: (((0 + s_0) + s_1) + ...)
    }
}

// sum over rows of (largest - smallest column): the plan's test whether rows
// reach across x (random columns) or stay near the diagonal (bands, stencils)
__global__ void row_span_kernel(int64_t nrows, const int* __restrict__ rp, const int* __restrict__ col,
                                unsigned long long* __restrict__ total) {
    unsigned long long acc = 0;
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < nrows; r += (int64_t)gridDim.x * blockDim.x) {
        int lo = INT32_MAX, hi = -1;
        for (int k = rp[r]; k < rp[r + 1]; ++k) { lo = min(lo, col[k]); hi = max(hi, col[k]); }
        if (hi >= lo) acc += (unsigned long long)(hi - lo);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if ((threadIdx.x & 31) == 0) atomicAdd(total, acc);
}

// entry positions k of the plan's CSR copy (k in [pad, pad + nnz)) ->
// slot k - pad: its panel key, its row, and k itself (the sort's payload)
__global__ void panel_keys_kernel(int64_t nrows, const int* __restrict__ rp, const int* __restrict__ col, int lg, int pad,
                                  unsigned char* __restrict__ key, int* __restrict__ row_of, int* __restrict__ idx) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < nrows; r += (int64_t)gridDim.x * blockDim.x)
        for (int k = rp[r]; k < rp[r + 1]; ++k) {
            key[k - pad] = (unsigned char)(col[k] >> lg);
            row_of[k - pad] = (int)r;
            idx[k - pad] = k;
        }
}
// sorted keys -> first position of each present panel
__global__ void panel_bounds_kernel(int64_t n, const unsigned char* __restrict__ skey, int64_t* __restrict__ zoff) {
    for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
        if (p == 0 || skey[p] != skey[p - 1]) zoff[skey[p]] = p;
}
// per panel k: the first pair whose entries start at or after zoff[k]
__global__ void panel_pair_offsets_kernel(int npanels, const int64_t* __restrict__ zoff, const int* __restrict__ pstart,
                                          int64_t npairs, int* __restrict__ poff) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k > npanels) return;
    int64_t lo = 0, hi = npairs;
    while (lo < hi) {
        const int64_t m = (lo + hi) / 2;
        if ((int64_t)pstart[m] < zoff[k]) lo = m + 1;
        else hi = m;
    }
    poff[k] = (int)lo;
}
template <typename T>
__global__ void panel_gather_kernel(int64_t n, int pad, const int* __restrict__ sidx, const int* __restrict__ col,
                                    const T* __restrict__ val, const int* __restrict__ row_of,
                                    const unsigned char* __restrict__ skey, int* __restrict__ pcol, T* __restrict__ pval,
                                    int* __restrict__ prow_full, unsigned char* __restrict__ head) {
    for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x) {
        const int k = sidx[p];
        pcol[p] = col[k];
        pval[p] = val[k];
        const int r = row_of[k - pad];
        prow_full[p] = r;
        head[p] = p == 0 || skey[p] != skey[p - 1] || row_of[sidx[p - 1] - pad] != r;
    }
}
__global__ void panel_pairs_kernel(int64_t npairs, const int* __restrict__ starts, const int* __restrict__ prow_full,
                                   int* __restrict__ prow) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < npairs; j += (int64_t)gridDim.x * blockDim.x)
        prow[j] = prow_full[starts[j]];
}

constexpr int kStreamVecFlag = 0x40000000;   // item.y flag: the item holds a row longer than VEC

template <int NB, int RMAX, typename T>
struct StreamStage {
    T val[NB + 8];
    int col[NB + 8];
    int rp[RMAX + 8];
};

template <int BLOCK, int STAGES, int NB, int RMAX, int VEC, typename T>
__global__ void __launch_bounds__(BLOCK) csr_stream_tma_kernel(int nitems, const int4* __restrict__ items,
                                                               const int* __restrict__ rp,
                                                               const int* __restrict__ col,
                                                               const T* __restrict__ val,
                                                               const T* __restrict__ x,
                                                               T* __restrict__ y,
                                                               T* __restrict__ carry) {
    using Stage = StreamStage<NB, RMAX, T>;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Stage* st = reinterpret_cast<Stage*>(smem_raw);
    __shared__ __align__(8) uint64_t full[STAGES];
    __shared__ T s_red[BLOCK / 32];

    const int tid = threadIdx.x;
    const int G = gridDim.x;
    const int nmine = nitems > (int)blockIdx.x ? (nitems - (int)blockIdx.x + G - 1) / G : 0;

    uint64_t pol = 0;
    if (tid == 0) {
        for (int s = 0; s < STAGES; ++s) mbar_init(&full[s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        pol = evict_first_policy();
    }
    __syncthreads();

    auto issue = [&](int j) {   // thread 0: stream local item j into stage j % STAGES
        const int4 it = __ldg(items + blockIdx.x + (int64_t)j * G);
        Stage& S = st[j % STAGES];
        const int k0a = it.z & ~3, k1a = (it.w + 3) & ~3;
        uint32_t bytes = (uint32_t)(k1a - k0a) * (uint32_t)(sizeof(T) + 4);
        int r0a = 0, r1a = 0;
        if (it.y >= 0) {
            const int r1 = it.y & ~kStreamVecFlag;
            r0a = it.x & ~3;
            r1a = (r1 + 1 + 3) & ~3;
            bytes += (uint32_t)(r1a - r0a) * 4u;
        }
        mbar_arrive_expect_tx(&full[j % STAGES], bytes);
        if (k1a > k0a) {
            tma_load_1d(S.val, val + k0a, (uint32_t)(k1a - k0a) * (uint32_t)sizeof(T), &full[j % STAGES], pol);
            tma_load_1d(S.col, col + k0a, (uint32_t)(k1a - k0a) * 4u, &full[j % STAGES], pol);
        }
        if (r1a > r0a) tma_load_1d(S.rp, rp + r0a, (uint32_t)(r1a - r0a) * 4u, &full[j % STAGES], pol);
    };

    if (tid == 0)
        for (int j = 0; j < STAGES - 1 && j < nmine; ++j) issue(j);

    for (int j = 0; j < nmine; ++j) {
        if (tid == 0 && j + STAGES - 1 < nmine) issue(j + STAGES - 1);
        const int4 it = __ldg(items + blockIdx.x + (int64_t)j * G);
        Stage& S = st[j % STAGES];
        mbar_wait(&full[j % STAGES], (uint32_t)((j / STAGES) & 1));

        const int k0a = it.z & ~3;
        const int off = it.z - k0a;
        const int nz = it.w - it.z;
        // phase 1: products in place, balanced over nonzeros. Batched: all of
        // a thread's (val, col) smem reads, then all its x gathers, then the
        // products, so the gathers overlap instead of forming a serial chain.
        {
            constexpr int PER = (NB + BLOCK - 1) / BLOCK;
            T v[PER];
            int c[PER];
#pragma unroll
            for (int u = 0; u < PER; ++u) {
                const int i = tid + u * BLOCK;
                v[u] = T(0);
                c[u] = 0;
                if (i < nz) { v[u] = S.val[off + i]; c[u] = S.col[off + i]; }
            }
            T xv[PER];
#pragma unroll
            for (int u = 0; u < PER; ++u) xv[u] = (tid + u * BLOCK < nz) ? ld_x_ordered(x, c[u]) : T(0);
#pragma unroll
            for (int u = 0; u < PER; ++u) {
                const int i = tid + u * BLOCK;
                if (i < nz) S.val[off + i] = v[u] * xv[u];
            }
        }
        __syncthreads();
        // phase 2: the reduction order is a property of the row alone (not of
        // the item it landed in), so results do not depend on item or rank
        // boundaries: rows of <= VEC entries are summed sequentially by one
        // thread (the oracle's order); longer rows lane-strided by a warp.
        if (it.y >= 0) {
            const bool has_long = (it.y & kStreamVecFlag) != 0;
            const int r0 = it.x, r1 = it.y & ~kStreamVecFlag, roff = r0 - (r0 & ~3);
            for (int r = tid; r < r1 - r0; r += BLOCK) {
                const int s = S.rp[roff + r] - k0a, e = S.rp[roff + r + 1] - k0a;
                if (e - s > VEC) continue;
                T acc = T(+0.0);
                for (int k = s; k < e; ++k) acc = acc + S.val[k];
                y[r0 + r] = acc;
            }
            if (has_long) {
                const int lane = tid & 31, w = tid >> 5;
                for (int r = w; r < r1 - r0; r += BLOCK / 32) {
                    const int s = S.rp[roff + r] - k0a, e = S.rp[roff + r + 1] - k0a;
                    if (e - s <= VEC) continue;
                    T acc = T(0);
                    for (int k = s + lane; k < e; k += 32) acc += S.val[k];
#pragma unroll
                    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
                    if (lane == 0) y[r0 + r] = acc;
                }
            }
        } else {
            // long-row piece: deterministic block sum -> carry slot
            T acc = T(0);
            for (int i = tid; i < nz; i += BLOCK) acc += S.val[off + i];
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
            if ((tid & 31) == 0) s_red[tid >> 5] = acc;
            __syncthreads();
            if (tid == 0) {
                T t = T(0);
                for (int w = 0; w < BLOCK / 32; ++w) t += s_red[w];
                carry[-it.y - 1] = t;
            }
        }
        __syncthreads();   // stage j is free; make generic-proxy writes visible to the async proxy
        if (tid == 0) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
}

// y[row] = sum of its long-row pieces: one warp per long row, lane-strided
// over the pieces then a fixed shuffle tree (deterministic)
template <typename T>
__global__ void csr_stream_fixup_kernel(int nlong, const int4* __restrict__ longrows, const T* __restrict__ carry,
                                        T* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int i = (int)((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    if (i >= nlong) return;
    const int4 L = longrows[i];   // (row, first piece, end piece, -)
    T s = T(0);
    for (int p = L.y + lane; p < L.z; p += 32) s += carry[p];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) y[L.x] = s;
}

// =====================================================================
// plan-time helpers
// =====================================================================
// validation + context statistics over the caller's int64 row pointer
struct RowStats {
    unsigned long long sum_len2_lo;   // Σ len^2 (wraps only beyond 2^64)
    unsigned long long max_len;
    unsigned long long empty;
    int bad;
};

__global__ void rowptr_check_narrow_kernel(int64_t nrows, const int64_t* __restrict__ rp64, int64_t first, int pad,
                                           int* __restrict__ rp32, RowStats* st) {
    unsigned long long s2 = 0, mx = 0, em = 0;
    int bad = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= nrows; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t v = rp64[i];
        rp32[i] = (int)(v - first + pad);
        if (i < nrows) {
            const int64_t len = rp64[i + 1] - v;
            if (len < 0) bad = 1;
            else {
                s2 += (unsigned long long)len * (unsigned long long)len;
                mx = max(mx, (unsigned long long)len);
                em += (len == 0);
            }
        }
    }
    // warp reduce then one atomic per warp
    for (int off = 16; off > 0; off >>= 1) {
        s2 += __shfl_xor_sync(0xffffffffu, s2, off);
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, off));
        em += __shfl_xor_sync(0xffffffffu, em, off);
        bad |= __shfl_xor_sync(0xffffffffu, bad, off);
    }
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(&st->sum_len2_lo, s2);
        atomicMax(&st->max_len, mx);
        atomicAdd(&st->empty, em);
        if (bad) atomicOr(&st->bad, 1);
    }
}

__global__ void col_check_kernel(int64_t n, const int* __restrict__ col, int64_t ncols, int* bad) {
    int b = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int c = col[i];
        b |= (c < 0 || (int64_t)c >= ncols);
    }
    b = __any_sync(0xffffffffu, b);
    if (b && (threadIdx.x & 31) == 0) atomicOr(bad, 1);
}

// SELL conversion -----------------------------------------------------
// key for the σ-window sort: (window, descending length, row) packed in 64 bits
// Rows longer than `cap` are left out of the SELL layout (length 0 there) and
// summed by sell_long_kernel instead (hybrid SELL for heavy-tailed rows).
__global__ void sell_keys_kernel(int nrows, const int* __restrict__ rp, int sigma, int maxlen, int cap,
                                 unsigned long long* __restrict__ keys, int* __restrict__ rows) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nrows) return;
    int len = rp[i + 1] - rp[i];
    if (len > cap) len = 0;
    const unsigned long long win = (unsigned long long)(i / sigma);
    keys[i] = (win << 32) | (unsigned long long)(maxlen - len);
    rows[i] = i;
}

// sorted position r -> original row perm[r]; lengths + per-chunk max
// chunk_len[c] = max length, | kSellMasked unless all 32 rows exist with that length
__global__ void sell_lengths_kernel(int nrows, const int* __restrict__ rp, const int* __restrict__ perm, int cap,
                                    int* __restrict__ rowlen, int* __restrict__ chunk_len) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    const int lane = threadIdx.x & 31;
    int len = -1;
    if (r < nrows) {
        const int o = perm ? perm[r] : r;
        len = rp[o + 1] - rp[o];
        if (len > cap) len = 0;
        rowlen[r] = len;
    }
    int mx = len, mn = len;
    for (int off = 16; off > 0; off >>= 1) {
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, off));
        mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, off));
    }
    mx = max(mx, 0);
    if (lane == 0 && r < nrows) chunk_len[r >> 5] = (mn == mx) ? mx : (mx | kSellMasked);
}

template <typename T>
__global__ void sell_fill_kernel(int nrows, const int* __restrict__ rp, const int* __restrict__ perm, int cap,
                                 const int* __restrict__ src_col, const T* __restrict__ src_val,
                                 const int64_t* __restrict__ chunk_ptr, int* __restrict__ col,
                                 T* __restrict__ val) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= nrows) return;
    const int o = perm ? perm[r] : r;
    const int s = rp[o], e = rp[o + 1];
    if (e - s > cap) return;   // a long row: sell_long_kernel's
    const int64_t base = chunk_ptr[r >> 5] + (r & 31);
    for (int k = s; k < e; ++k) {
        col[base + (int64_t)(k - s) * 32] = src_col[k];
        val[base + (int64_t)(k - s) * 32] = src_val[k];
    }
}

// Long rows of a hybrid SELL plan (length > cap): segments of up to
// kSellLongSeg nonzeros, one CTA per segment (seg = {row, k begin, k end,
// long-row index}; lrow = {first segment, segment count}). Each thread sums a
// strided subsequence of the segment (coalesced val / col streams, 4 loads
// in flight), the CTA reduces in a fixed tree, thread 0 stores the segment's
// partial; the CTA that completes a row's last segment (per-row counter,
// reset for the next call) adds the row's partials in segment order and
// writes y. No fp atomics: the result does not depend on scheduling.
// Launched after sell_kernel, which wrote 0 for these rows.
constexpr int kSellLongSeg = 4096;
template <int BLOCK, typename T>
__global__ void __launch_bounds__(BLOCK) sell_long_kernel(const int4* __restrict__ seg, const int2* __restrict__ lrow,
                                                          unsigned int* __restrict__ cnt, T* __restrict__ part,
                                                          const int* __restrict__ col, const T* __restrict__ val,
                                                          const T* __restrict__ x, T* __restrict__ y) {
    constexpr int NW = BLOCK / 32;
    __shared__ T s_w[NW];
    __shared__ bool s_last;
    const int4 g = seg[blockIdx.x];
    const uint64_t pol = evict_first_policy();
    T a0 = T(0), a1 = T(0), a2 = T(0), a3 = T(0);
    int k = g.y + threadIdx.x;
    for (; k + 3 * BLOCK < g.z; k += 4 * BLOCK) {
        const int c0 = ld_stream_i(col + k, pol), c1 = ld_stream_i(col + k + BLOCK, pol);
        const int c2 = ld_stream_i(col + k + 2 * BLOCK, pol), c3 = ld_stream_i(col + k + 3 * BLOCK, pol);
        const T v0 = ld_stream_v(val + k, pol), v1 = ld_stream_v(val + k + BLOCK, pol);
        const T v2 = ld_stream_v(val + k + 2 * BLOCK, pol), v3 = ld_stream_v(val + k + 3 * BLOCK, pol);
        a0 = fma(v0, ld_x(x, c0), a0);
        a1 = fma(v1, ld_x(x, c1), a1);
        a2 = fma(v2, ld_x(x, c2), a2);
        a3 = fma(v3, ld_x(x, c3), a3);
    }
    for (; k < g.z; k += BLOCK) a0 = fma(ld_stream_v(val + k, pol), ld_x(x, ld_stream_i(col + k, pol)), a0);
    T acc = (a0 + a1) + (a2 + a3);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if ((threadIdx.x & 31) == 0) s_w[threadIdx.x >> 5] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        T t = s_w[0];
#pragma unroll
        for (int w = 1; w < NW; ++w) t += s_w[w];
        part[blockIdx.x] = t;
        __threadfence();
        const int2 lr = lrow[g.w];
        s_last = atomicAdd(cnt + g.w, 1u) == (unsigned)(lr.y - 1);
        if (s_last) {
            __threadfence();
            T r = T(0);
            for (int j = 0; j < lr.y; ++j) r += __ldcg(part + lr.x + j);
            y[g.x] = r;
            cnt[g.w] = 0u;
        }
    }
}

// Mid-length rows of a hybrid SELL plan (cap < length <= kSellLongSeg): one
// warp per listed row, lanes strided over the row (4 col / val pairs, then 4
// x gathers in flight per lane), a fixed-order shuffle reduction, lane 0
// writes y — no scratch, deterministic. Launched after sell_kernel, which
// wrote 0 for these rows.
template <int BLOCK, typename T>
__global__ void __launch_bounds__(BLOCK) sell_mid_kernel(int n, const int* __restrict__ rows,
                                                         const int* __restrict__ rp, const int* __restrict__ col,
                                                         const T* __restrict__ val, const T* __restrict__ x,
                                                         T* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int w = (blockIdx.x * BLOCK + threadIdx.x) >> 5;
    if (w >= n) return;
    const int r = __ldg(rows + w);
    const int s = __ldg(rp + r), e = __ldg(rp + r + 1);
    const uint64_t pol = evict_first_policy();
    T a0 = T(0), a1 = T(0), a2 = T(0), a3 = T(0);
    int k = s + lane;
    for (; k + 96 < e; k += 128) {
        const int c0 = ld_stream_i(col + k, pol), c1 = ld_stream_i(col + k + 32, pol);
        const int c2 = ld_stream_i(col + k + 64, pol), c3 = ld_stream_i(col + k + 96, pol);
        const T v0 = ld_stream_v(val + k, pol), v1 = ld_stream_v(val + k + 32, pol);
        const T v2 = ld_stream_v(val + k + 64, pol), v3 = ld_stream_v(val + k + 96, pol);
        a0 = fma(v0, ld_x(x, c0), a0);
        a1 = fma(v1, ld_x(x, c1), a1);
        a2 = fma(v2, ld_x(x, c2), a2);
        a3 = fma(v3, ld_x(x, c3), a3);
    }
    for (; k < e; k += 32) a0 = fma(ld_stream_v(val + k, pol), ld_x(x, ld_stream_i(col + k, pol)), a0);
    T acc = (a0 + a1) + (a2 + a3);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) y[r] = acc;
}

// 16-bit column deltas: one warp per chunk; if every stored column of the
// chunk is within int16 of its row's original index, write col16 and set
// kSellCol16 in chunk_len.
__global__ void sell_col16_kernel(int nrows, int nchunks, const int64_t* __restrict__ chunk_ptr,
                                  int* __restrict__ chunk_len, const int* __restrict__ rowlen,
                                  const int* __restrict__ perm, const int* __restrict__ col,
                                  int16_t* __restrict__ col16, unsigned long long* __restrict__ n16) {
    const int lane = threadIdx.x & 31;
    const int c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (c >= nchunks) return;
    const int d = chunk_len[c];
    if (d & (kSellStencil | kSellPattern)) return;   // already needs no column stream
    const int clen = d & kSellLenMask;
    const int r = c * 32 + lane;
    const int len = r < nrows ? rowlen[r] : 0;
    const int orow = (perm && r < nrows) ? perm[r] : r;
    const int64_t base = chunk_ptr[c] + lane;
    bool ok = true;
    for (int j = 0; j < len; ++j) {
        const int dl = col[base + (int64_t)j * 32] - orow;
        ok &= (dl >= -32768 && dl <= 32767);
    }
    ok = __all_sync(0xffffffffu, ok);
    if (!ok) return;
    for (int j = 0; j < clen; ++j)
        col16[base + (int64_t)j * 32] = (int16_t)(j < len ? col[base + (int64_t)j * 32] - orow : 0);
    if (lane == 0) {
        chunk_len[c] = d | kSellCol16;
        atomicAdd(n16, 1ull);
    }
}

// Stencil chunks: one warp per chunk; a uniform chunk (all 32 rows present,
// all of length clen) whose slot-j column offsets (col - row) are equal in
// every lane stores those clen offsets once: soff[chunk_ptr[c]/32 + j].
__device__ __forceinline__ bool bits_equal(double a, double b) { return __double_as_longlong(a) == __double_as_longlong(b); }
__device__ __forceinline__ bool bits_equal(float a, float b) { return __float_as_int(a) == __float_as_int(b); }

template <typename T>
__global__ void sell_stencil_kernel(int nrows, int nchunks, const int64_t* __restrict__ chunk_ptr,
                                    int* __restrict__ chunk_len, const int* __restrict__ perm,
                                    const int* __restrict__ col, int* __restrict__ soff,
                                    unsigned long long* __restrict__ nst,
                                    const T* __restrict__ val, T* __restrict__ sconst,
                                    unsigned char* __restrict__ cflag, unsigned long long* __restrict__ nconst) {
    const int lane = threadIdx.x & 31;
    const int c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (c >= nchunks) return;
    const int d = chunk_len[c];
    if (d & kSellMasked) return;        // rows of different lengths (or a partial chunk)
    const int clen = d & kSellLenMask;
    if (clen > 32) return;              // the kernel keeps slot offsets one per lane
    const int r = c * 32 + lane;
    const int orow = perm ? perm[r] : r;
    const int64_t base = chunk_ptr[c] + lane;
    bool same = true;
    for (int j = 0; j < clen; ++j) {
        const int dl = col[base + (int64_t)j * 32] - orow;
        same &= dl == __shfl_sync(0xffffffffu, dl, 0);
    }
    if (!__all_sync(0xffffffffu, same)) return;
    const int64_t sb = chunk_ptr[c] >> 5;
    for (int j = lane; j < clen; j += 32) soff[sb + j] = col[chunk_ptr[c] + (int64_t)j * 32] - (perm ? perm[c * 32] : c * 32);
    // value compression (sconst != nullptr): every slot's 32 values bitwise
    // identical -> one value per slot, the value stream is never read
    bool cval = sconst != nullptr;
    for (int j = 0; cval && j < clen; ++j) {
        const T v = val[base + (int64_t)j * 32];
        cval = __all_sync(0xffffffffu, bits_equal(v, __shfl_sync(0xffffffffu, v, 0)));
    }
    // constant chunk: cflag[c] = 1 and sconst[sb + j] = slot j's value (the
    // plan dedupes (offsets, values) into its pattern table on the host)
    if (cval)
        for (int j = lane; j < clen; j += 32) sconst[sb + j] = val[chunk_ptr[c] + (int64_t)j * 32];
    if (cflag && lane == 0) cflag[c] = cval ? 1 : 0;
    if (lane == 0) {
        chunk_len[c] = d | kSellStencil;
        atomicAdd(nst, 1ull);
        if (cval) atomicAdd(nconst, 1ull);
    }
}

// halo pack / unpack --------------------------------------------------
template <typename T>
__global__ void gather_kernel(int64_t n, const int* __restrict__ idx, const T* __restrict__ src,
                              T* __restrict__ dst) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] = src[idx[i]];
}
// union row pointer of shipped row blocks (distribution candidates): a
// block's narrowed row pointer (local offsets + its alignment pad) widened
// and moved to the union's nonzero offset: out[i] = rp[i] + delta
__global__ void rowptr_widen_kernel(int64_t n, const int* __restrict__ rp, int64_t delta, int64_t* __restrict__ out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (int64_t)rp[i] + delta;
}
template <typename T>
__global__ void scatter_kernel(int64_t n, const int* __restrict__ idx, const T* __restrict__ src,
                               T* __restrict__ dst) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[idx[i]] = src[i];
}


// =====================================================================
// Fused compute + halo exchange over peer memory (exchange PEPP_X_P2P).
// One kernel per partitioned iteration computes the rows the neighbours read
// (the head [0, h) and tail [R - t, R) of the block), stores each result in
// the local y AND straight into every receiving peer's copy of the same
// buffer (CUDA-IPC mapped peer memory: NVLink / NVSwitch stores), then
// signals the peers with release stores to flags in their memory and waits
// (acquire) until every peer this rank receives from has signalled. Replaces
// head/tail SpMV kernels + NCCL send/recv + pack/unpack of the in-order path.
//
// Protocol (per plan, `epoch` e = number of P2P calls so far, device
// resident so CUDA graphs replay it correctly). Each rank's signal block
// holds ready[P] and arrive[P], one slot per peer:
//   my.ready[q]  = e+1 : rank q (which RECEIVES from me) began call e, so
//                        everything q's streams did before (calls < e, which
//                        read q's buffers — e.g. the previous x — and the
//                        caller's own writes, e.g. filling x_0) is complete:
//                        I may now write into q's y of call e;
//   my.arrive[q] = e+1 : rank q (which SENDS to me) has landed its rows of
//                        call e in my y.
// Readiness flows from receiver to sender and data + arrival from sender to
// receiver, so the send and receive peer sets need not match (nonsymmetric
// matrices: upwind stencils, one-sided bands). Call e on rank r: every CTA
// writes ready = e+1 into the block of each rank r receives from
// (idempotent; no CTA waits for another CTA of the grid), waits for
// my.ready[q] >= e+1 from every rank q r sends to, computes its rows and
// pushes them; the last CTA (grid-wide counter) fences, writes arrive = e+1
// into each send-peer's block, waits for my.arrive[q] >= e+1 from every
// receive-peer, resets the counter and bumps the epoch. Kernel completion
// therefore means exactly what the NCCL halo's stream completion means: own
// rows and every ghost are in y. Deadlock freedom: call e waits only for
// the peers' call e (ready: published first thing; arrive: published after
// their own ready waits, which depend only on call e starting everywhere),
// and call e starts after call e-1 completed — by induction on e, no cycle.
// Every wait is bounded (%globaltimer, timeout_ns: 20 s, PEPP_P2P_TIMEOUT_MS): a peer that never
// arrives sets *err (host-mapped) instead of hanging the GPU.
//
// Row sums are the oracle's arithmetic (sequential in CSR order, product
// rounded then sum rounded: __dmul_rn / __dadd_rn, no FMA), one thread per
// row: boundary rows of stencils / banded matrices are short.
// =====================================================================
constexpr int kP2PMaxPeers = 8;
constexpr int kP2PMaxPush = 16;

template <typename T>
struct P2PArgs {
    int64_t seg_lo[2], seg_hi[2];      // local rows computed here: head, tail
    int64_t row_offset;                // global index of local row 0
    int npush;                         // push ranges: local rows [lo, hi) -> peer buffer base
    int64_t push_lo[kP2PMaxPush], push_hi[kP2PMaxPush];
    T* push_dst[kP2PMaxPush];          // the peer's buffer (global indexing)
    int nsend;                         // peers this rank writes to
    unsigned long long* ready_in[kP2PMaxPeers];      // &my.ready[send peer]       (waited on)
    unsigned long long* arrive_out[kP2PMaxPeers];    // &send_peer.arrive[me]      (published)
    int nrecv;                         // peers this rank receives from
    unsigned long long* ready_out[kP2PMaxPeers];     // &recv_peer.ready[me]       (published)
    unsigned long long* arrive_in[kP2PMaxPeers];     // &my.arrive[recv peer]      (waited on)
    unsigned long long* epoch;         // my signal block
    unsigned int* done;                // my signal block: CTAs finished this call
    int* err;                          // host-mapped error flag
    unsigned long long timeout_ns;     // bound on every wait
};

__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long global_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// spin until *p >= v (bounded); false on timeout
__device__ __forceinline__ bool wait_geq(const unsigned long long* p, unsigned long long v, unsigned long long t0,
                                         unsigned long long timeout_ns) {
    while (ld_acquire_sys(p) < v) {
        if (global_ns() - t0 > timeout_ns) return false;
        __nanosleep(64);
    }
    return true;
}

__device__ __forceinline__ double mul_rn(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ double add_rn(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ float mul_rn(float a, float b) { return __fmul_rn(a, b); }
__device__ __forceinline__ float add_rn(float a, float b) { return __fadd_rn(a, b); }

template <typename T>
__global__ void __launch_bounds__(256) halo_push_kernel(const int* __restrict__ rp, const int* __restrict__ col,
                                                        const T* __restrict__ val, const T* __restrict__ x,
                                                        T* __restrict__ y, const __grid_constant__ P2PArgs<T> a) {
    __shared__ unsigned long long s_epoch;
    __shared__ int s_last;
    const unsigned long long t0 = global_ns();
    if (threadIdx.x == 0) {
        const unsigned long long e = *(volatile unsigned long long*)a.epoch;
        s_epoch = e;
        for (int j = 0; j < a.nrecv; ++j) st_release_sys(a.ready_out[j], e + 1);
        bool ok = true;
        for (int j = 0; j < a.nsend; ++j) ok &= wait_geq(a.ready_in[j], e + 1, t0, a.timeout_ns);
        if (!ok) atomicExch(a.err, 1);
    }
    __syncthreads();
    const int64_t n0 = a.seg_hi[0] - a.seg_lo[0], n = n0 + (a.seg_hi[1] - a.seg_lo[1]);
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = t < n0 ? a.seg_lo[0] + t : a.seg_lo[1] + (t - n0);
        T acc = T(0);
        for (int k = rp[i]; k < rp[i + 1]; ++k) acc = add_rn(acc, mul_rn(val[k], x[col[k]]));
        const int64_t g = a.row_offset + i;
        y[g] = acc;
        for (int j = 0; j < a.npush; ++j)
            if (i >= a.push_lo[j] && i < a.push_hi[j]) a.push_dst[j][g] = acc;
    }
    // publish: every CTA's stores before the last CTA's arrive flags
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) s_last = atomicAdd(a.done, 1u) == gridDim.x - 1;
    __syncthreads();
    if (!s_last || threadIdx.x != 0) return;
    __threadfence_system();
    const unsigned long long e = s_epoch;
    for (int j = 0; j < a.nsend; ++j) st_release_sys(a.arrive_out[j], e + 1);
    bool ok = true;
    for (int j = 0; j < a.nrecv; ++j) ok &= wait_geq(a.arrive_in[j], e + 1, global_ns(), a.timeout_ns);
    if (!ok) atomicExch(a.err, 1);
    *a.done = 0u;
    *(volatile unsigned long long*)a.epoch = e + 1;
    __threadfence();
}

}  // namespace k
}  // namespace pepp
