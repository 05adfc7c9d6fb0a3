// ws_sell_probe.cu — standalone experiment (round 2): can a warp-specialized
// SELL kernel beat the LDG form on a gather-bound matrix (config 2's shape)?
// The random-column SELL walk is bound by the L1 -> XBAR sector requests
// (DESIGN.md §6): the x gathers AND the value / column streams go through
// the LSU. Here one producer warp per CTA streams each chunk's columns and
// values into a shared-memory ring with cp.async.bulk (TMA: no LSU sector
// requests), and 15 consumer warps only gather x from L2 and do the FMAs.
// Round 1's probe of a TMA ring (gather_stream_probe.cu) used 2 CTAs x 8
// warps that both streamed and gathered, and lost to occupancy (94 vs 80 us).
//
// Config 2: 2^20 rows x 2^20 columns, 16 distinct random columns per row
// (SELL-32, σ = 1, column-major chunks: slot j of lane l at chunk*512 + j*32 + l).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 ws_sell_probe.cu -o ws_sell_probe
//
// Measured on one B200 (round 2; results equal to the LDG kernel's):
//   LDG warp-per-chunk                   75.2 us
//   WS 15 consumers, 24 stages, 1 CTA/SM 73.8 us
//   WS 15 consumers, 32 stages, 1 CTA/SM 78.5 us
//   WS 31 consumers, 32 stages, 1 CTA/SM 80.2 us
//   WS  7 consumers, 12 stages, 2 CTA/SM 74.8 us
// Taking the value / column streams off the LSU gains 2 % at best: the x
// gathers themselves hold the ceiling (68.5 us with no streams at all,
// gather_stream_probe.cu). Not worth restructuring SELL around.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>

constexpr int L = 16;          // slots per chunk
constexpr int CH = 32 * L;     // entries per chunk

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
    uint32_t done;
    do {
        asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
                     : "=r"(done) : "r"(smem_u32(b)), "r"(parity) : "memory");
    } while (!done);
}
__device__ __forceinline__ void bulk(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

// baseline: warp per chunk, all loads through the LSU (the library's walk, minus its pipelining)
__global__ void __launch_bounds__(256) ldg_sell(int nchunks, const int* __restrict__ col, const double* __restrict__ val,
                                                const double* __restrict__ x, double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    for (int c = (blockIdx.x * 256 + threadIdx.x) >> 5; c < nchunks; c += (gridDim.x * 256) >> 5) {
        int ci[L];
        double v[L], xv[L];
#pragma unroll
        for (int j = 0; j < L; ++j) {
            ci[j] = __ldg(col + (size_t)c * CH + j * 32 + lane);
            v[j] = __ldg(val + (size_t)c * CH + j * 32 + lane);
        }
#pragma unroll
        for (int j = 0; j < L; ++j) xv[j] = __ldg(x + ci[j]);
        double acc = 0;
#pragma unroll
        for (int j = 0; j < L; ++j) acc = fma(v[j], xv[j], acc);
        y[c * 32 + lane] = acc;
    }
}

template <int NC, int S>
__global__ void __launch_bounds__(32 * (NC + 1), 1) ws_sell(int nchunks, const int* __restrict__ col,
                                                            const double* __restrict__ val,
                                                            const double* __restrict__ x, double* __restrict__ y) {
    extern __shared__ __align__(128) unsigned char sm[];
    double* sval = reinterpret_cast<double*>(sm);                      // [S][CH]
    int* scol = reinterpret_cast<int*>(sm + (size_t)S * CH * 8);       // [S][CH]
    __shared__ __align__(8) uint64_t full[S], empty[S];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int c0 = (int)((int64_t)nchunks * blockIdx.x / gridDim.x), c1 = (int)((int64_t)nchunks * (blockIdx.x + 1) / gridDim.x);
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (warp == 0) {   // producer
        if (lane == 0)
            for (int c = c0, k = 0; c < c1; ++c, ++k) {
                const int s = k % S;
                if (k >= S) mbar_wait(&empty[s], (uint32_t)((k / S) - 1) & 1u);
                mbar_expect(&full[s], CH * 12);
                bulk(sval + (size_t)s * CH, val + (size_t)c * CH, CH * 8, &full[s]);
                bulk(scol + (size_t)s * CH, col + (size_t)c * CH, CH * 4, &full[s]);
            }
        return;
    }
    const int cw = warp - 1;
    for (int c = c0 + cw, k = cw; c < c1; c += NC, k += NC) {
        const int s = k % S;
        mbar_wait(&full[s], (uint32_t)(k / S) & 1u);
        int ci[L];
        double v[L], xv[L];
#pragma unroll
        for (int j = 0; j < L; ++j) { ci[j] = scol[(size_t)s * CH + j * 32 + lane]; v[j] = sval[(size_t)s * CH + j * 32 + lane]; }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[s]);   // the stage's data is in registers
#pragma unroll
        for (int j = 0; j < L; ++j) xv[j] = __ldg(x + ci[j]);
        double acc = 0;
#pragma unroll
        for (int j = 0; j < L; ++j) acc = fma(v[j], xv[j], acc);
        y[c * 32 + lane] = acc;
    }
}

template <typename F>
float timeit(F f) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    f();
    cudaEventRecord(a);
    for (int r = 0; r < 10; ++r) f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    return ms / 10 * 1000.f;
}

int main() {
    setvbuf(stdout, nullptr, _IONBF, 0);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int R = 1 << 20, nchunks = R / 32;
    const size_t nnz = (size_t)R * L;
    std::vector<int> hc(nnz);
    std::vector<double> hv(nnz), hx(R);
    std::mt19937_64 g(42);
    for (int c = 0; c < nchunks; ++c)
        for (int l = 0; l < 32; ++l) {
            std::vector<int> cs;
            while ((int)cs.size() < L) {
                const int v = (int)(g() % R);
                if (std::find(cs.begin(), cs.end(), v) == cs.end()) cs.push_back(v);
            }
            std::sort(cs.begin(), cs.end());
            for (int j = 0; j < L; ++j) {
                hc[(size_t)c * CH + j * 32 + l] = cs[j];
                hv[(size_t)c * CH + j * 32 + l] = (double)((int)(g() % 9) - 4);
            }
        }
    for (auto& v : hx) v = (double)((int)(g() % 17) - 8);
    int* col;
    double *val, *x, *y1, *y2;
    cudaMalloc(&col, nnz * 4);
    cudaMalloc(&val, nnz * 8);
    cudaMalloc(&x, R * 8);
    cudaMalloc(&y1, R * 8);
    cudaMalloc(&y2, R * 8);
    cudaMemcpy(col, hc.data(), nnz * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(val, hv.data(), nnz * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(x, hx.data(), R * 8, cudaMemcpyHostToDevice);
    const float t0 = timeit([&] { ldg_sell<<<sms * 8, 256>>>(nchunks, col, val, x, y1); });
    printf("LDG warp-per-chunk              : %7.1f us\n", t0);
    auto run = [&](auto kern, int nc, int stages, int ctas) {
        const size_t smem = (size_t)stages * CH * 12;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        const float t = timeit([&] { kern<<<sms * ctas, 32 * (nc + 1), smem>>>(nchunks, col, val, x, y2); });
        cudaError_t e = cudaDeviceSynchronize();
        std::vector<double> a(R), b(R);
        cudaMemcpy(a.data(), y1, R * 8, cudaMemcpyDeviceToHost);
        cudaMemcpy(b.data(), y2, R * 8, cudaMemcpyDeviceToHost);
        printf("WS %2d consumers, %2d stages, %d CTA/SM: %7.1f us  (%s)%s\n", nc, stages, ctas, t, a == b ? "equal" : "DIFFER",
               e == cudaSuccess ? "" : cudaGetErrorString(e));
    };
    run(ws_sell<15, 24>, 15, 24, 1);
    run(ws_sell<15, 32>, 15, 32, 1);
    run(ws_sell<31, 32>, 31, 32, 1);
    run(ws_sell<7, 12>, 7, 12, 2);   // (stages must be >= consumers: a stage is handed to one consumer at a time)
    return 0;
}
