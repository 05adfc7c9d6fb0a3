// gather_stream_probe.cu — standalone experiment (not part of the library):
// on a gather-bound SELL matrix (BASELINE config 2 shape: 1M x 1M, 16 random
// columns per row, uniform chunks of 16 slots), does the val / col STREAM
// compete with the x GATHERS for the SM's L1 -> XBAR request interface? If
// so, feeding val / col through the TMA (cp.async.bulk into shared memory)
// frees that interface for the gathers.
//   ldg        : warp per chunk, 16 col + 16 val loads per lane (coalesced),
//                16 gathers, 16 FMAs (the library's SELL inner loop)
//   gather_only: the same gathers and FMAs, columns from a hash, no streams
//   tma        : persistent CTAs; thread 0 bulk-copies each group of 8 chunks
//                (8 x 32 x 16 x 12 B = 48 KB) into a 2-stage smem ring (2 CTAs per SM), warp w
//                computes chunk w of the group from shared memory (LDS) and
//                gathers x with LDG
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a gather_stream_probe.cu -o gsp
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)
constexpr int R = 1 << 20;   // rows = cols
constexpr int S = 16;        // slots per chunk
constexpr int NCH = R / 32;
constexpr int G = 8;         // chunks per TMA group (one per warp)
constexpr int STAGES = 2;
constexpr int GROUP_BYTES = G * 32 * S * 12;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t* b, int n) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(n)); }
__device__ __forceinline__ void mb_expect(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mb_arrive(uint64_t* b) { asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory"); }
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
__device__ __forceinline__ int ldi(const int* p, uint64_t pol) { int r; asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol)); return r; }

// layout per chunk c: col[c][S][32] int32 then (separate array) val[c][S][32] double
__global__ void __launch_bounds__(256) k_ldg(const int* __restrict__ col, const double* __restrict__ val,
                                             const double* __restrict__ x, double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int nw = (gridDim.x * 256) >> 5;
    const uint64_t pol = pol_ef();
    for (int c = (blockIdx.x * 256 + threadIdx.x) >> 5; c < NCH; c += nw) {
        const int64_t b = (int64_t)c * S * 32 + lane;
        int ci[S];
        double v[S], xv[S];
#pragma unroll
        for (int j = 0; j < S; ++j) ci[j] = ldi(col + b + j * 32, pol);
#pragma unroll
        for (int j = 0; j < S; ++j) v[j] = ldd(val + b + j * 32, pol);
#pragma unroll
        for (int j = 0; j < S; ++j) xv[j] = __ldg(x + ci[j]);
        double acc = 0;
#pragma unroll
        for (int j = 0; j < S; ++j) acc = fma(v[j], xv[j], acc);
        y[c * 32 + lane] = acc;
    }
}

__device__ __forceinline__ uint32_t hsh(uint32_t a) { a ^= a >> 16; a *= 0x7feb352du; a ^= a >> 15; a *= 0x846ca68bu; a ^= a >> 16; return a; }

__global__ void __launch_bounds__(256) k_gather_only(const double* __restrict__ x, double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int nw = (gridDim.x * 256) >> 5;
    for (int c = (blockIdx.x * 256 + threadIdx.x) >> 5; c < NCH; c += nw) {
        const int r = c * 32 + lane;
        double xv[S];
#pragma unroll
        for (int j = 0; j < S; ++j) xv[j] = __ldg(x + (hsh(r * S + j) & (R - 1)));
        double acc = 0;
#pragma unroll
        for (int j = 0; j < S; ++j) acc = fma(0.5, xv[j], acc);
        y[r] = acc;
    }
}

// persistent: CTA b owns groups b, b + grid, ...; group = G consecutive chunks.
// smem stage = G chunks of cols (G*S*32*4) then G chunks of vals (G*S*32*8)
__global__ void __launch_bounds__(256) k_tma(const int* __restrict__ col, const double* __restrict__ val,
                                             const double* __restrict__ x, double* __restrict__ y) {
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t full[STAGES], empty[STAGES];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int ngroups = NCH / G;
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) { mb_init(&full[s], 1); mb_init(&empty[s], 8); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto issue = [&](int g, int s) {
        unsigned char* st = smem + s * GROUP_BYTES;
        const int64_t c0 = (int64_t)g * G;
        mb_expect(&full[s], GROUP_BYTES);
        bulk(st, col + c0 * S * 32, G * S * 32 * 4, &full[s]);
        bulk(st + G * S * 32 * 4, val + c0 * S * 32, G * S * 32 * 8, &full[s]);
    };
    int it = 0;
    if (threadIdx.x == 0)
        for (int s = 0; s < STAGES; ++s) {
            const int g = blockIdx.x + s * gridDim.x;
            if (g < ngroups) issue(g, s);
        }
    for (int g = blockIdx.x; g < ngroups; g += gridDim.x, ++it) {
        const int s = it % STAGES;
        const uint32_t ph = (it / STAGES) & 1;
        mb_wait(&full[s], ph);
        const unsigned char* st = smem + s * GROUP_BYTES;
        const int* sc = (const int*)st + w * S * 32;
        const double* sv = (const double*)(st + G * S * 32 * 4) + w * S * 32;
        int ci[S];
        double v[S], xv[S];
#pragma unroll
        for (int j = 0; j < S; ++j) { ci[j] = sc[j * 32 + lane]; v[j] = sv[j * 32 + lane]; }
        __syncwarp();
        if (lane == 0) mb_arrive(&empty[s]);   // this warp is done with the stage's smem
#pragma unroll
        for (int j = 0; j < S; ++j) xv[j] = __ldg(x + ci[j]);
        double acc = 0;
#pragma unroll
        for (int j = 0; j < S; ++j) acc = fma(v[j], xv[j], acc);
        y[((int64_t)g * G + w) * 32 + lane] = acc;
        if (threadIdx.x == 0) {   // refill this stage once all 8 warps released it
            const int gn = g + STAGES * gridDim.x;
            if (gn < ngroups) { mb_wait(&empty[s], ph); issue(gn, s); }
        }
    }
}

int main() {
    std::vector<int> hc((size_t)R * S);
    std::vector<double> hv((size_t)R * S), hx(R);
    uint64_t st = 42;
    auto rnd = [&]() { st ^= st << 13; st ^= st >> 7; st ^= st << 17; return st; };
    for (auto& c : hc) c = (int)(rnd() & (R - 1));
    for (auto& v : hv) v = (double)(rnd() % 1000) / 1000.0;
    for (auto& v : hx) v = (double)(rnd() % 1000) / 1000.0;
    int *dc; double *dv, *dx, *dy, *dflush;
    CK(cudaMalloc(&dc, sizeof(int) * hc.size()));
    CK(cudaMalloc(&dv, sizeof(double) * hv.size()));
    CK(cudaMalloc(&dx, sizeof(double) * R));
    CK(cudaMalloc(&dy, sizeof(double) * R));
    CK(cudaMalloc(&dflush, 512 << 20));
    CK(cudaMemcpy(dc, hc.data(), sizeof(int) * hc.size(), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dv, hv.data(), sizeof(double) * hv.size(), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dx, hx.data(), sizeof(double) * R, cudaMemcpyHostToDevice));
    int sms = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    const int smem = STAGES * GROUP_BYTES;
    CK(cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    int occ_tma = 0, occ_ldg = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_tma, k_tma, 256, smem));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_ldg, k_ldg, 256, 0));
    printf("sms %d occ_ldg %d occ_tma %d (smem %d B)\n", sms, occ_ldg, occ_tma, smem);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    auto timeit = [&](const char* name, auto launch) {
        float best = 1e9, sum = 0;
        const int reps = 20;
        for (int r = 0; r < reps + 2; ++r) {
            cudaMemsetAsync(dflush, r, 512 << 20);
            cudaEventRecord(a);
            launch();
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (r >= 2) { best = ms < best ? ms : best; sum += ms; }
        }
        printf("%-12s best %8.2f us  mean %8.2f us  (%.1f G gathers/s)\n", name, best * 1e3, sum / reps * 1e3,
               (double)R * S / (best * 1e-3) / 1e9);
    };
    std::vector<double> y1(R), y2(R);
    timeit("ldg", [&] { k_ldg<<<sms * occ_ldg, 256>>>(dc, dv, dx, dy); });
    CK(cudaMemcpy(y1.data(), dy, sizeof(double) * R, cudaMemcpyDeviceToHost));
    timeit("gather_only", [&] { k_gather_only<<<sms * occ_ldg, 256>>>(dx, dy); });
    for (int grid_mult : {1, 2}) {
        if (grid_mult > occ_tma) break;
        char nm[32];
        snprintf(nm, sizeof nm, "tma x%d", grid_mult);
        timeit(nm, [&] { k_tma<<<sms * grid_mult, 256, smem>>>(dc, dv, dx, dy); });
    }
    CK(cudaGetLastError());
    CK(cudaMemcpy(y2.data(), dy, sizeof(double) * R, cudaMemcpyDeviceToHost));
    int bad = 0;
    for (int i = 0; i < R; ++i) bad += y1[i] != y2[i];
    printf("tma vs ldg mismatches: %d\n", bad);
    return 0;
}
