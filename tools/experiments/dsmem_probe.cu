// dsmem_probe.cu — standalone experiment: can distributed shared memory
// raise the random-gather ceiling of SpMV with random columns (BASELINE
// configs 2 and 3)? Global gathers are capped at ~1 sector request per
// SM-cycle on the L1->XBAR interface. Here each CTA of a
// cluster holds one slice of x in shared memory; gathers whose column falls
// in the cluster's slices are served over DSMEM (ld.shared::cluster), the
// rest from L2. Indices are streamed coalesced (4 B each), as in the SpMV.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 dsmem_probe.cu -o dsmem_probe
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ uint32_t cta_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ double ld_dsmem(uint32_t local_addr, uint32_t rank) {
    uint32_t ra;
    double v;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(local_addr), "r"(rank));
    asm volatile("ld.shared::cluster.f64 %0, [%1];" : "=d"(v) : "r"(ra));
    return v;
}

// MODE 0: every gather from global (L2); 1: columns < CL*S from DSMEM (local
// slice included), the rest from global; 2: every gather from DSMEM
// (column mod CL*S); 3: every gather from the CTA's own slice (column mod S).
template <int MODE, int ILP>
__global__ void __launch_bounds__(1024, 1) probe(int64_t n, const int* __restrict__ idx, const double* __restrict__ x,
                                                  int S, int CL, double* __restrict__ out) {
    extern __shared__ double s_x[];
    const uint32_t rank = cta_rank();
    if (MODE != 0) {
        for (int i = threadIdx.x; i < S; i += blockDim.x) s_x[i] = x[(int64_t)rank * S + i];
        cluster_sync();
    }
    const uint32_t sbase = smem_u32(s_x);
    const int lane = threadIdx.x & 31;
    const int64_t W = (int64_t)gridDim.x * (blockDim.x >> 5);
    const int64_t w = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    const int64_t b0 = w * n / W, b1 = (w + 1) * n / W;
    const int span = CL * S;
    double acc = 0;
    for (int64_t b = b0; b < b1; b += 32 * ILP) {
        int c[ILP];
#pragma unroll
        for (int u = 0; u < ILP; ++u) {
            const int64_t i = b + u * 32 + lane;
            c[u] = i < b1 ? __ldg(idx + i) : -1;
        }
        double v[ILP];
#pragma unroll
        for (int u = 0; u < ILP; ++u) {
            int cc = c[u];
            if (cc < 0) { v[u] = 0; continue; }
            if (MODE == 0) v[u] = __ldg(x + cc);
            else if (MODE == 1) {
                if (cc < span) { const int r = cc / S; v[u] = ld_dsmem(sbase + 8u * (uint32_t)(cc - r * S), r); }
                else v[u] = __ldg(x + cc);
            } else if (MODE == 2) {
                cc %= span;
                const int r = cc / S;
                v[u] = ld_dsmem(sbase + 8u * (uint32_t)(cc - r * S), r);
            } else {
                v[u] = s_x[cc % S];
            }
        }
#pragma unroll
        for (int u = 0; u < ILP; ++u) acc += v[u];
    }
    if (acc == 1234.5) out[0] = acc;
    if (MODE != 0) cluster_sync();   // no CTA leaves while others may read its slice
}

template <int MODE, int ILP>
void run(const char* name, int64_t n, const int* idx, const double* x, double* out, int CL, int S, int nblk) {
    auto k = probe<MODE, ILP>;
    const size_t smem = MODE == 0 ? 0 : (size_t)S * 8;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CL; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cfg.blockDim = dim3(1024);
    cfg.dynamicSmemBytes = smem;
    cfg.attrs = at; cfg.numAttrs = 1;
    int ncl = 0;
    cfg.gridDim = dim3(CL);
    if (cudaOccupancyMaxActiveClusters(&ncl, k, &cfg) != cudaSuccess || ncl == 0) {
        printf("  %-26s CL=%2d: cannot be resident (%s)\n", name, CL, cudaGetErrorString(cudaGetLastError()));
        return;
    }
    const int grid = nblk > 0 ? nblk : ncl * CL;
    cfg.gridDim = dim3(grid);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaLaunchKernelEx(&cfg, k, n, idx, x, S, CL, out);
    cudaEventRecord(a);
    for (int r = 0; r < 5; ++r) cudaLaunchKernelEx(&cfg, k, n, idx, x, S, CL, out);
    cudaEventRecord(b); cudaEventSynchronize(b);
    cudaError_t e = cudaGetLastError();
    float ms; cudaEventElapsedTime(&ms, a, b);
    const double t = ms / 5 * 1e-3;
    printf("  %-26s CL=%2d ILP=%2d S=%6d clusters=%3d grid=%4d: %8.1f us %6.1f G/s (%.2f per SM-cycle @1.965GHz) %s\n",
           name, CL, ILP, S, ncl, grid, t * 1e6, n / t / 1e9, n / t / (148 * 1.965e9), e ? cudaGetErrorString(e) : "");
}

int main() {
    const int64_t n = 16LL << 20;   // 16.8M gathers (config 2's nnz)
    const int S = 24576;            // 192 KB slice per CTA
    for (int64_t xs : {1LL << 20, 4LL << 20}) {
        std::vector<int> h(n);
        std::mt19937_64 g(7);
        for (auto& v : h) v = (int)(g() % xs);
        int* idx; double *x, *out;
        cudaMalloc(&idx, n * 4); cudaMalloc(&x, xs * 8); cudaMalloc(&out, 8);
        cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice);
        cudaMemset(x, 0, xs * 8);
        printf("x = %lld doubles (%lld MB)\n", (long long)xs, (long long)(xs * 8 >> 20));
        run<0, 8>("global only", n, idx, x, out, 1, S, 148);
        run<0, 16>("global only", n, idx, x, out, 1, S, 148);
        run<3, 8>("local smem only", n, idx, x, out, 1, S, 148);
        for (int CL : {2, 4, 8, 16}) {
            run<2, 8>("dsmem only", n, idx, x, out, CL, S, 0);
            run<2, 16>("dsmem only", n, idx, x, out, CL, S, 0);
            run<1, 8>("split dsmem/global", n, idx, x, out, CL, S, 0);
            run<1, 16>("split dsmem/global", n, idx, x, out, CL, S, 0);
        }
        cudaFree(idx); cudaFree(x); cudaFree(out);
    }
    return 0;
}
