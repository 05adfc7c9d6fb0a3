// tma_probe.cu — standalone experiment (not part of the library): how fast can
// a cp.async.bulk (TMA) shared-memory ring stream CSR val/col on B200, and what
// does each phase of the CSR-stream kernel cost on top of it?
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tma_probe.cu -o tma_probe
//   ./tma_probe            (Laplacian-like column pattern, 335M nnz, fp64)
//
// mode 0: LDG.128 grid-stride read of val+col (read-only streaming ceiling)
// mode 1: TMA ring, consumers touch one smem word per item      (TMA ceiling)
// mode 2: TMA ring + phase 1 (x gathers, products to smem)
// mode 3: mode 2 + a per-row-like reduction (every 5 products summed, stored)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)

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

__global__ void ldg_stream(int64_t n, const double* __restrict__ val, const int* __restrict__ col, double* out) {
    double acc = 0;
    int64_t n4 = n / 4;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
        int4 c = __ldg(reinterpret_cast<const int4*>(col) + i);
        double2 a = __ldg(reinterpret_cast<const double2*>(val) + 2 * i);
        double2 b = __ldg(reinterpret_cast<const double2*>(val) + 2 * i + 1);
        acc += a.x + a.y + b.x + b.y + c.x + c.y + c.z + c.w;
    }
    if (acc == 12345.678) out[0] = acc;
}

template <int BLOCK, int STAGES, int NB, int MODE>
__global__ void __launch_bounds__(BLOCK) tma_ring(int nitems, const double* __restrict__ val, const int* __restrict__ col,
                                                  const double* __restrict__ x, double* __restrict__ y) {
    extern __shared__ __align__(128) unsigned char sm[];
    double* sval = reinterpret_cast<double*>(sm);                       // [STAGES][NB]
    int* scol = reinterpret_cast<int*>(sm + sizeof(double) * NB * STAGES);
    __shared__ __align__(8) uint64_t full[STAGES];
    const int tid = threadIdx.x, G = gridDim.x;
    const int nmine = nitems > (int)blockIdx.x ? (nitems - (int)blockIdx.x + G - 1) / G : 0;
    if (tid == 0) {
        for (int s = 0; s < STAGES; ++s) mb_init(&full[s]);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto issue = [&](int j) {
        const int64_t it = blockIdx.x + (int64_t)j * G;
        const int s = j % STAGES;
        mb_expect(&full[s], NB * 12);
        bulk(sval + s * NB, val + it * NB, NB * 8, &full[s]);
        bulk(scol + s * NB, col + it * NB, NB * 4, &full[s]);
    };
    if (tid == 0)
        for (int j = 0; j < STAGES - 1 && j < nmine; ++j) issue(j);
    double keep = 0;
    for (int j = 0; j < nmine; ++j) {
        if (tid == 0 && j + STAGES - 1 < nmine) issue(j + STAGES - 1);
        const int s = j % STAGES;
        mb_wait(&full[s], (j / STAGES) & 1);
        double* v = sval + s * NB;
        const int* c = scol + s * NB;
        const int64_t it = blockIdx.x + (int64_t)j * G;
        if (MODE == 1) {
            keep += v[tid];
        } else {
            constexpr int PER = NB / BLOCK;
            double xv[PER], vv[PER];
#pragma unroll
            for (int u = 0; u < PER; ++u) { vv[u] = v[tid + u * BLOCK]; xv[u] = __ldg(x + c[tid + u * BLOCK]); }
#pragma unroll
            for (int u = 0; u < PER; ++u) v[tid + u * BLOCK] = vv[u] * xv[u];
            if (MODE == 3) {
                __syncthreads();
                for (int r = tid; r < NB / 5; r += BLOCK) {
                    double a = 0;
                    for (int k = 0; k < 5; ++k) a += v[r * 5 + k];
                    y[it * (NB / 5) + r] = a;
                }
            }
        }
        __syncthreads();
        if (tid == 0) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    if (keep == 12345.678) y[0] = keep;
}

template <int BLOCK, int STAGES, int NB, int MODE>
float run_ring(int sms, int nitems, const double* val, const int* col, const double* x, double* y) {
    auto k = tma_ring<BLOCK, STAGES, NB, MODE>;
    size_t smem = (size_t)STAGES * NB * 12;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, BLOCK, smem);
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    k<<<sms * occ, BLOCK, smem>>>(nitems, val, col, x, y);
    cudaEventRecord(a);
    for (int r = 0; r < 5; ++r) k<<<sms * occ, BLOCK, smem>>>(nitems, val, col, x, y);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("  ring BLOCK=%d STAGES=%d NB=%d MODE=%d occ=%d: %.1f us  -> %.0f GB/s (val+col)\n", BLOCK, STAGES, NB, MODE,
           occ, ms * 1000 / 5, (double)nitems * NB * 12 / (ms / 5 * 1e-3) / 1e9);
    return ms / 5;
}

int main() {
    const int64_t n = 8192LL * 8192 * 5;   // ~335M "nnz"
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    double *val, *x, *y;
    int* col;
    CK(cudaMalloc(&val, n * 8));
    CK(cudaMalloc(&col, n * 4));
    CK(cudaMalloc(&x, 8192LL * 8192 * 8));
    CK(cudaMalloc(&y, 8192LL * 8192 * 8));
    CK(cudaMemset(val, 0, n * 8));
    CK(cudaMemset(x, 0, 8192LL * 8192 * 8));
    {   // Laplacian-like columns: nnz k of row r=k/5 -> r-8192, r-1, r, r+1, r+8192 (clamped)
        std::vector<int> h(n);
        const int64_t R = 8192LL * 8192;
        for (int64_t k = 0; k < n; ++k) {
            int64_t r = k / 5, d = k % 5;
            int64_t c = d == 0 ? r - 8192 : d == 1 ? r - 1 : d == 2 ? r : d == 3 ? r + 1 : r + 8192;
            h[k] = (int)(c < 0 ? 0 : c >= R ? R - 1 : c);
        }
        CK(cudaMemcpy(col, h.data(), n * 4, cudaMemcpyHostToDevice));
    }
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    ldg_stream<<<sms * 8, 256>>>(n, val, col, y);
    cudaEventRecord(a);
    for (int r = 0; r < 5; ++r) ldg_stream<<<sms * 8, 256>>>(n, val, col, y);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("ldg_stream: %.1f us -> %.0f GB/s (val+col)\n", ms * 1000 / 5, n * 12.0 / (ms / 5 * 1e-3) / 1e9);
    const int n25 = (int)(n / 2560);   // items of 2560 nnz (= 512 rows of 5)
    run_ring<256, 2, 2560, 1>(sms, n25, val, col, x, y);
    run_ring<256, 3, 2560, 1>(sms, n25, val, col, x, y);
    run_ring<256, 4, 2560, 1>(sms, n25, val, col, x, y);
    run_ring<256, 2, 2560, 2>(sms, n25, val, col, x, y);
    run_ring<256, 3, 2560, 2>(sms, n25, val, col, x, y);
    run_ring<256, 2, 2560, 3>(sms, n25, val, col, x, y);
    run_ring<256, 3, 2560, 3>(sms, n25, val, col, x, y);
    const int n51 = (int)(n / 5120);
    run_ring<512, 2, 5120, 1>(sms, n51, val, col, x, y);
    run_ring<512, 2, 5120, 2>(sms, n51, val, col, x, y);
    run_ring<512, 3, 5120, 3>(sms, n51, val, col, x, y);
    const int n12 = (int)(n / 1280);
    run_ring<128, 2, 1280, 1>(sms, n12, val, col, x, y);
    run_ring<128, 3, 1280, 2>(sms, n12, val, col, x, y);
    run_ring<128, 4, 1280, 3>(sms, n12, val, col, x, y);
    run_ring<128, 6, 1280, 3>(sms, n12, val, col, x, y);
    CK(cudaDeviceSynchronize());
    return 0;
}
