// gather_probe.cu — standalone experiment: random 8-byte gather throughput on
// B200 (the bound of SpMV with random columns, BASELINE configs 2 and 3).
// Indices are streamed coalesced (4 B each); x is gathered at random.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 gather_probe.cu -o gather_probe
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <cuda_runtime.h>

template <int MODE, int ILP>
__global__ void __launch_bounds__(256) gather(int64_t n, const int* __restrict__ idx, const double* __restrict__ x,
                                              double* __restrict__ out) {
    double acc = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x * ILP;
    for (int64_t b = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x); b < n; b += stride) {
        int c[ILP];
#pragma unroll
        for (int u = 0; u < ILP; ++u) {
            const int64_t i = b + (int64_t)u * gridDim.x * blockDim.x;
            c[u] = i < n ? __ldg(idx + i) : 0;
        }
        double v[ILP];
#pragma unroll
        for (int u = 0; u < ILP; ++u) {
            if (MODE == 0) v[u] = __ldg(x + c[u]);
            else if (MODE == 1) asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v[u]) : "l"(x + c[u]));
            else asm volatile("ld.global.cg.f64 %0, [%1];" : "=d"(v[u]) : "l"(x + c[u]));
        }
#pragma unroll
        for (int u = 0; u < ILP; ++u) acc += v[u];
    }
    if (acc == 1234.5) out[0] = acc;
}

template <int MODE, int ILP>
void run(const char* name, int64_t n, const int* idx, const double* x, double* out, int grid) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    gather<MODE, ILP><<<grid, 256>>>(n, idx, x, out);
    cudaEventRecord(a);
    for (int r = 0; r < 5; ++r) gather<MODE, ILP><<<grid, 256>>>(n, idx, x, out);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    const double t = ms / 5 * 1e-3;
    printf("  %-22s ILP=%d grid=%6d: %8.1f us  %6.1f G gathers/s  (%.2f per SM-cycle @1.965GHz)\n", name, ILP, grid, t * 1e6,
           n / t / 1e9, n / t / (148 * 1.965e9));
}

int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int64_t n = 16LL << 20;   // 16.8M gathers (config 2's nnz)
    for (int64_t xs : {1LL << 20, 4LL << 20, 64LL << 20}) {
        std::vector<int> h(n);
        std::mt19937_64 g(7);
        for (auto& v : h) v = (int)(g() % xs);
        int* idx; double *x, *out;
        cudaMalloc(&idx, n * 4); cudaMalloc(&x, xs * 8); cudaMalloc(&out, 8);
        cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice);
        cudaMemset(x, 0, xs * 8);
        printf("x = %lld doubles (%lld MB)\n", (long long)xs, (long long)(xs * 8 >> 20));
        run<0, 4>("ldg (L1 allocate)", n, idx, x, out, sms * 8);
        run<0, 8>("ldg (L1 allocate)", n, idx, x, out, sms * 8);
        run<0, 16>("ldg (L1 allocate)", n, idx, x, out, sms * 8);
        run<1, 8>("nc.L1::no_allocate", n, idx, x, out, sms * 8);
        run<1, 16>("nc.L1::no_allocate", n, idx, x, out, sms * 8);
        run<2, 8>("cg (L2 only)", n, idx, x, out, sms * 8);
        run<2, 16>("cg (L2 only)", n, idx, x, out, sms * 8);
        cudaFree(idx); cudaFree(x); cudaFree(out);
    }
    return 0;
}
