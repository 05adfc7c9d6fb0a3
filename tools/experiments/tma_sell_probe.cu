// tma_sell_probe.cu — standalone experiment (not part of the library): can a
// TMA-fed SELL beat the library's register-pipelined LDG SELL on the config-4
// Laplacian? Layout as in the library's stencil chunks: per chunk of 32 rows,
// 5 value slots (column-major, 32 doubles per slot) and one set of 5 column
// offsets for the whole chunk; x gathered at row + offset; y written.
//   ldg : one warp per chunk, grid-stride, chunk i+1's offsets prefetched
//   tma : persistent CTAs own contiguous chunk groups; one thread streams each
//         group's values (G chunks x 1280 B) into a STAGES-deep smem ring with
//         cp.async.bulk; warp w of the CTA computes chunk w of each group.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)
constexpr int N = 8192;
constexpr int S = 5;   // slots per chunk

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t* b) { asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(b))); }
__device__ __forceinline__ void mb_expect(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mb_wait(uint64_t* b, uint32_t ph) {
    uint32_t d;
    do {
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                     : "=r"(d) : "r"(su32(b)), "r"(ph) : "memory");
    } while (!d);
}
__device__ __forceinline__ void bulk(void* dst, const void* src, uint32_t n, uint64_t* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(su32(dst)), "l"(src), "r"(n), "r"(su32(b)) : "memory");
}
__device__ __forceinline__ uint64_t pol_ef() { uint64_t p; asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ double ldd(const double* p, uint64_t pol) { double r; asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(r) : "l"(p), "l"(pol)); return r; }

__global__ void __launch_bounds__(256) sell_ldg(int nchunks, const int* __restrict__ off, const double* __restrict__ val,
                                                const double* __restrict__ x, double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int warp = (blockIdx.x * 256 + threadIdx.x) >> 5;
    const int nw = (gridDim.x * 256) >> 5;
    const uint64_t pol = pol_ef();
    int c = warp;
    int o = (c < nchunks && lane < S) ? __ldg(off + c * S + lane) : 0;
    for (; c < nchunks; c += nw) {
        const int cn = c + nw;
        const int on = (cn < nchunks && lane < S) ? __ldg(off + cn * S + lane) : 0;
        const int r = c * 32 + lane;
        double v[S], xv[S];
#pragma unroll
        for (int j = 0; j < S; ++j) v[j] = ldd(val + (int64_t)c * 32 * S + j * 32 + lane, pol);
#pragma unroll
        for (int j = 0; j < S; ++j) {
            int col = r + __shfl_sync(0xffffffffu, o, j);
            col = col < 0 ? 0 : (col >= N * N ? N * N - 1 : col);
            xv[j] = __ldg(x + col);
        }
        double acc = 0;
#pragma unroll
        for (int j = 0; j < S; ++j) acc = fma(v[j], xv[j], acc);
        y[r] = acc;
        o = on;
    }
}

template <int WARPS, int STAGES, int G>
__global__ void __launch_bounds__(WARPS * 32) sell_tma(int ngroups, const int* __restrict__ off, const double* __restrict__ val,
                                                       const double* __restrict__ x, double* __restrict__ y) {
    static_assert(G == WARPS, "one warp per chunk of a group");
    extern __shared__ __align__(128) double ring[];   // [STAGES][G * 32 * S]
    __shared__ __align__(8) uint64_t full[STAGES];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const int Gd = gridDim.x;
    const int nmine = ngroups > (int)blockIdx.x ? (ngroups - (int)blockIdx.x + Gd - 1) / Gd : 0;
    constexpr uint32_t bytes = G * 32 * S * 8;
    if (tid == 0) {
        for (int s = 0; s < STAGES; ++s) mb_init(&full[s]);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto issue = [&](int j) {
        const int64_t g = blockIdx.x + (int64_t)j * Gd;
        mb_expect(&full[j % STAGES], bytes);
        bulk(ring + (size_t)(j % STAGES) * G * 32 * S, val + g * G * 32 * S, bytes, &full[j % STAGES]);
    };
    if (tid == 0)
        for (int j = 0; j < STAGES - 1 && j < nmine; ++j) issue(j);
    for (int j = 0; j < nmine; ++j) {
        if (tid == 0 && j + STAGES - 1 < nmine) issue(j + STAGES - 1);
        const int64_t g = blockIdx.x + (int64_t)j * Gd;
        const int c = (int)(g * G + w);
        const int r = c * 32 + lane;
        // x gathers need only the offsets: issue them before waiting for the values
        const int o = lane < S ? __ldg(off + c * S + lane) : 0;
        double xv[S];
#pragma unroll
        for (int jj = 0; jj < S; ++jj) {
            int col = r + __shfl_sync(0xffffffffu, o, jj);
            col = col < 0 ? 0 : (col >= N * N ? N * N - 1 : col);
            xv[jj] = __ldg(x + col);
        }
        mb_wait(&full[j % STAGES], (j / STAGES) & 1);
        const double* v = ring + (size_t)(j % STAGES) * G * 32 * S + w * 32 * S;
        double acc = 0;
#pragma unroll
        for (int jj = 0; jj < S; ++jj) acc = fma(v[jj * 32 + lane], xv[jj], acc);
        y[r] = acc;
        __syncthreads();   // stage free before it is refilled
    }
}

template <int WARPS, int STAGES>
void run_tma(int sms, int nchunks, const int* off, const double* val, const double* x, double* y) {
    auto k = sell_tma<WARPS, STAGES, WARPS>;
    size_t smem = (size_t)STAGES * WARPS * 32 * S * 8;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, WARPS * 32, smem);
    const int ngroups = nchunks / WARPS;
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    k<<<sms * occ, WARPS * 32, smem>>>(ngroups, off, val, x, y);
    cudaEventRecord(a);
    for (int i = 0; i < 10; ++i) k<<<sms * occ, WARPS * 32, smem>>>(ngroups, off, val, x, y);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    const double bytes = (double)nchunks * 32 * (S * 8 + 16);   // val + x + y (offsets negligible)
    printf("tma WARPS=%d STAGES=%d occ=%d smem=%zu: %.1f us  %.0f GB/s actual  %s\n", WARPS, STAGES, occ, smem, ms * 100,
           bytes / (ms / 10 * 1e-3) / 1e9, cudaGetErrorString(cudaGetLastError()));
}

int main() {
    const int64_t R = (int64_t)N * N;
    const int nchunks = (int)(R / 32);
    std::vector<int> off((size_t)nchunks * S);
    for (int c = 0; c < nchunks; ++c) { const int o[S] = {-N, -1, 0, 1, N}; for (int j = 0; j < S; ++j) off[(size_t)c * S + j] = o[j]; }
    int* doff; double *dval, *dx, *dy;
    CK(cudaMalloc(&doff, off.size() * 4)); CK(cudaMalloc(&dval, (size_t)nchunks * 32 * S * 8));
    CK(cudaMalloc(&dx, R * 8)); CK(cudaMalloc(&dy, R * 8));
    CK(cudaMemcpy(doff, off.data(), off.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemset(dval, 0, (size_t)nchunks * 32 * S * 8)); CK(cudaMemset(dx, 0, R * 8));
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int g : {sms * 8, sms * 6}) {
        cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
        sell_ldg<<<g, 256>>>(nchunks, doff, dval, dx, dy);
        cudaEventRecord(a);
        for (int i = 0; i < 10; ++i) sell_ldg<<<g, 256>>>(nchunks, doff, dval, dx, dy);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        printf("ldg grid=%d: %.1f us  %.0f GB/s actual\n", g, ms * 100, (double)nchunks * 32 * (S * 8 + 16) / (ms / 10 * 1e-3) / 1e9);
    }
    run_tma<8, 2>(sms, nchunks, doff, dval, dx, dy);
    run_tma<8, 3>(sms, nchunks, doff, dval, dx, dy);
    run_tma<8, 4>(sms, nchunks, doff, dval, dx, dy);
    run_tma<8, 6>(sms, nchunks, doff, dval, dx, dy);
    run_tma<16, 3>(sms, nchunks, doff, dval, dx, dy);
    run_tma<16, 4>(sms, nchunks, doff, dval, dx, dy);
    run_tma<4, 4>(sms, nchunks, doff, dval, dx, dy);
    run_tma<4, 8>(sms, nchunks, doff, dval, dx, dy);
    CK(cudaDeviceSynchronize());
    return 0;
}
