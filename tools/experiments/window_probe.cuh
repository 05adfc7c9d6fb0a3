// window_probe.cuh — ROUND-2 EXPERIMENT, NOT BUILT INTO THE LIBRARY.
//
// Value-compressed SELL (pattern chunks) through a per-SM shared-memory
// window of x, as it was measured on config 4 (8192^2 Laplacian, fp64,
// compress_values = 1) inside plan.cu before being reverted:
//   list walk (sell_kernel phase A, the library's path)      254 us
//   window, one-thread cp.async.bulk (TMA) per 8 KB block    549-678 us
//   window, all-thread 16-byte cp.async, 5 blocks ahead      471 us
// The 5-point stencil's offsets span 16384 entries (two grid rows): in
// fp64 the window alone takes 128 KB of the SM's shared memory, leaving room
// for only ~40 KB of x in flight per SM — ~5x too little to cover DRAM
// latency at the copy rate (ncu: 50 % of warp samples at the tile barrier,
// long-scoreboard ~0: the warps wait for the ring, not for their own loads).
// Kept for the record; needs kernels.cuh's mbarrier / bulk
// copy helpers and SellPatterns to compile.
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// =====================================================================
// Value-compressed SELL through a shared-memory window of x (σ = 1 plans
// whose pattern chunks — offsets + values in the pattern table — dominate;
// the library-default layout of constant-coefficient stencils, config 4).
// The pattern chunks read only x and write y, and neighbouring rows read
// overlapping x (a 5-point stencil reads every x entry 5 times), so the
// L2-resident gathers of the list walk (phase A of sell_kernel: ~5 L1/L2
// requests per row, 0.66 of the copy peak, latency-bound at 1.2 eligible
// warps) are replaced by a per-SM window: each CTA (one per SM) owns a
// contiguous range of 1024-row tiles and streams x through a ring of K
// blocks of 1024 entries with cp.async.bulk (TMA, one mbarrier per slot):
// tile t needs blocks t .. t+nb-1 (nb covers the patterns' offset span),
// the ring holds K = nb + D of them, so D blocks load ahead while the tile
// computes, and block t's slot takes block t+K once tile t is done. x
// leaves DRAM once per CTA range (+ one span), y is written once. Rows are
// the pattern chunks of the tile (chunk_len flags; other chunks belong to
// the genlist walk, which runs beside this kernel); each row sums the same
// products in the same slot order as phase A (bit-identical). Blocks that
// would leave [0, ncols) are not loaded: tiles needing them read x from
// global memory directly.
// =====================================================================
constexpr int kWinRows = 1024;   // rows per tile = entries per ring block
constexpr int kWinBlock = 256;   // 8 warps x kWinCPW chunks per tile
constexpr int kWinCPW = 4;
constexpr int kWinMaxK = 64;
constexpr int kWinGuard = 32;    // ring[W, W+32) mirrors ring[0, 32): a warp's 32-row reads never wrap

template <int N, typename T, bool SMEM>
__device__ __forceinline__ T sell_window_row(const SellPatterns<T>& pt, int pid, const T* __restrict__ ring, int relm,
                                             int W, const T* __restrict__ x, int r) {
    T xv[N];
#pragma unroll
    for (int j = 0; j < N; ++j) {
        const int o = pt.off[pid][j];
        if (SMEM) {
            int q = relm + o;
            q += q < 0 ? W : 0;
            q -= q >= W ? W : 0;
            xv[j] = ring[q];
        } else {
            xv[j] = __ldg(x + r + o);
        }
    }
    T acc = T(0);
#pragma unroll
    for (int j = 0; j < N; ++j) acc = fma(pt.val[pid][j], xv[j], acc);   // slot order = the row's CSR order
    return acc;
}

template <typename T, bool SMEM>
__device__ __forceinline__ T sell_window_dispatch(int len, const SellPatterns<T>& pt, int pid, const T* __restrict__ ring,
                                                  int relm, int W, const T* __restrict__ x, int r) {
    switch (len) {
    case 1: return sell_window_row<1, T, SMEM>(pt, pid, ring, relm, W, x, r);
    case 2: return sell_window_row<2, T, SMEM>(pt, pid, ring, relm, W, x, r);
    case 3: return sell_window_row<3, T, SMEM>(pt, pid, ring, relm, W, x, r);
    case 4: return sell_window_row<4, T, SMEM>(pt, pid, ring, relm, W, x, r);
    case 5: return sell_window_row<5, T, SMEM>(pt, pid, ring, relm, W, x, r);
    case 6: return sell_window_row<6, T, SMEM>(pt, pid, ring, relm, W, x, r);
    case 7: return sell_window_row<7, T, SMEM>(pt, pid, ring, relm, W, x, r);
    default: return sell_window_row<8, T, SMEM>(pt, pid, ring, relm, W, x, r);
    }
}

struct WinMeta {                 // a tile's chunk descriptors, streamed with its last x block
    int64_t ptr[32];
    int len[32];
};

// N = the slots of the plan's dominant pattern `dom` (the one most chunks
// use): its offsets and values live in registers for the whole kernel, and a
// warp whose kWinCPW chunks of the tile all use it (and whose reads do not
// wrap the ring) takes the fast path — per chunk N shared-memory loads at
// immediate offsets, N FMAs and one store; any other chunk takes the
// general per-row path.
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait(int n) {   // all but the n most recent groups complete
    switch (n) {
    case 0: asm volatile("cp.async.wait_group 0;" ::: "memory"); break;
    case 1: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
    case 2: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
    case 3: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
    case 4: asm volatile("cp.async.wait_group 4;" ::: "memory"); break;
    case 5: asm volatile("cp.async.wait_group 5;" ::: "memory"); break;
    case 6: asm volatile("cp.async.wait_group 6;" ::: "memory"); break;
    default: asm volatile("cp.async.wait_group 7;" ::: "memory"); break;
    }
}

// N = the slots of the plan's dominant pattern `dom` (the one most chunks
// use): its offsets and values live in registers for the whole kernel, and a
// warp whose kWinCPW chunks of the tile all use it (and whose reads do not
// wrap the ring) takes the fast path — per chunk N shared-memory loads, N
// FMAs and one store; any other chunk takes the general per-row path. The
// ring is filled by every thread with 16-byte cp.async copies, one commit
// group per block (measured: one-thread cp.async.bulk (TMA) copies of the
// same blocks kept too few bytes in flight — ~5 µs per 8 KB copy under
// load, 549 µs on config 4, ncu: 50 % of warp samples at the tile barrier).
template <int N, typename T>
__global__ void __launch_bounds__(kWinBlock, 1) sell_window_kernel(int nrows, int ncols, int nchunks,
                                                                   const int* __restrict__ chunk_len,
                                                                   const int64_t* __restrict__ chunk_ptr,
                                                                   const __grid_constant__ SellPatterns<T> pt, int dom,
                                                                   const T* __restrict__ x, T* __restrict__ y,
                                                                   int K, int nb, int min_off) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    T* ring = reinterpret_cast<T*>(smem_raw);
    WinMeta* meta = reinterpret_cast<WinMeta*>(smem_raw + ((size_t)K * kWinRows + kWinGuard) * sizeof(T));
    constexpr int TR = kWinRows;
    constexpr int E16 = 16 / (int)sizeof(T);          // entries per 16-byte copy
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int ntiles = (nrows + TR - 1) / TR;
    const int t0 = (int)((int64_t)ntiles * blockIdx.x / gridDim.x);
    const int t1 = (int)((int64_t)ntiles * (blockIdx.x + 1) / gridDim.x);
    if (t0 >= t1) return;
    const int W = K * TR, D = K - nb;
    // global x index of ring block 0, floored to a multiple of 32, so a
    // chunk's 32 rows sit in one 32-aligned run of the ring
    int64_t base = (int64_t)t0 * TR + min_off;
    base = base >= 0 ? base / 32 * 32 : -((-base + 31) / 32 * 32);
    const int64_t ncols_al = (int64_t)ncols / 4 * 4;   // whole 16-byte units
    const int nt = t1 - t0, nblk = nt + nb;
    auto block_ok = [&](int b) {
        const int64_t g0 = base + (int64_t)b * TR;
        return g0 >= 0 && g0 + TR <= ncols_al;
    };
    // block b: x[base + b TR, +TR) (when inside x; slot 0 also fills the
    // guard) and the descriptors of tile b - nb + 1, the first tile that
    // needs it as its last block; one commit group per block on every thread
    auto issue = [&](int b) {
        if (b < nblk) {
            const int s = b % K, tile = b - nb + 1;
            if (block_ok(b)) {
                const T* src = x + base + (int64_t)b * TR;
                for (int i = tid; i < TR / E16; i += kWinBlock) cp_async16(ring + s * TR + i * E16, src + i * E16);
                if (s == 0 && tid < kWinGuard / E16) cp_async16(ring + W + tid * E16, src + tid * E16);
            }
            if (tile >= 0 && tile < nt) {
                const int64_t c0 = (int64_t)(t0 + tile) * 32;   // chunk_len / chunk_ptr are padded by 32 entries
                if (tid < 16) cp_async16(meta[s].ptr + 2 * tid, chunk_ptr + c0 + 2 * tid);
                else if (tid < 24) cp_async16(meta[s].len + 4 * (tid - 16), chunk_len + c0 + 4 * (tid - 16));
            }
        }
        cp_async_commit();
    };
    for (int b = 0; b < K; ++b) issue(b);
    int o[N];
    T v[N];
#pragma unroll
    for (int j = 0; j < N; ++j) { o[j] = pt.off[dom][j]; v[j] = pt.val[dom][j]; }
    // ring position of the tile's first row, (R0 - base) mod W (a multiple of
    // 32), advanced by TR per tile (no integer division in the loop)
    int rel0 = (int)(((int64_t)t0 * TR - base) % W);
    for (int t = 0; t < nt; ++t, rel0 = rel0 + TR >= W ? rel0 + TR - W : rel0 + TR) {
        cp_async_wait(D);                 // this thread's copies of blocks <= t + nb - 1 have landed
        __syncthreads();                  // ... and every other thread's
        const bool smem = block_ok(t) && block_ok(t + nb - 1);
        const WinMeta& M = meta[(t + nb - 1) % K];
        const int64_t R0 = (int64_t)(t0 + t) * TR;
        const int cw = warp * kWinCPW;                  // this warp's first chunk within the tile
        const int c0 = (int)(R0 >> 5) + cw;
        int w0 = rel0 + cw * 32;                        // ring position of the warp's first row
        w0 -= w0 >= W ? W : 0;
        bool fast = smem && c0 + kWinCPW <= nchunks;
#pragma unroll
        for (int u = 0; u < kWinCPW; ++u)
            fast &= (M.len[cw + u] & (kSellPattern | kSellLenMask)) == (kSellPattern | N) && (int)M.ptr[cw + u] == dom;
        const T* rp[N];                                 // per slot: the warp's run of the ring, linear
#pragma unroll
        for (int j = 0; j < N; ++j) {
            int q = w0 + o[j];
            q += q < 0 ? W : 0;
            q -= q >= W ? W : 0;
            fast &= q + kWinCPW * 32 <= W + kWinGuard;
            rp[j] = ring + q + lane;
        }
        if (fast) {
            T xv[kWinCPW][N];
#pragma unroll
            for (int u = 0; u < kWinCPW; ++u)
#pragma unroll
                for (int j = 0; j < N; ++j) xv[u][j] = rp[j][u * 32];
            T* yw = y + (int64_t)c0 * 32 + lane;
#pragma unroll
            for (int u = 0; u < kWinCPW; ++u) {
                T acc = T(0);
#pragma unroll
                for (int j = 0; j < N; ++j) acc = fma(v[j], xv[u][j], acc);   // slot order = the row's CSR order
                yw[u * 32] = acc;
            }
        } else {
#pragma unroll 1
            for (int u = 0; u < kWinCPW; ++u) {
                const int cl = cw + u, c = c0 + u;
                if (c >= nchunks) break;
                const int d = M.len[cl];
                if (!(d & kSellPattern)) continue;          // the genlist walk's chunk
                const int pid = (int)M.ptr[cl];
                const int r = c * 32 + lane;
                int relm = w0 + u * 32 + lane;
                relm -= relm >= W ? W : 0;
                y[r] = smem ? sell_window_dispatch<T, true>(d & kSellLenMask, pt, pid, ring, relm, W, x, r)
                            : sell_window_dispatch<T, false>(d & kSellLenMask, pt, pid, ring, relm, W, x, r);
            }
        }
        __syncthreads();                     // every thread is done with block t (and its descriptors)
        issue(t + K);
    }
}

