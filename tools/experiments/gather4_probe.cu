// gather4_probe.cu — standalone experiment (round 2): can
// the Blackwell tensor-map gather (cp.async.bulk.tensor.2d ... tile::gather4:
// one TMA instruction fetches 4 arbitrary rows of a 2D tensor into shared
// memory) beat the ~255 G/s ceiling of random 8-byte LDG gathers from an
// L2-resident x (gather_probe.cu; limiter: one L1->XBAR sector request per
// SM-cycle)? Config 2's shape: 16.8 M random columns into x of 2^20 doubles
// (8 MB, L2-resident), plus 4 M and 64 M-entry x.
//
// x is viewed as a 2D tensor of 16-byte rows (2 doubles), so gather4 with a
// {2, 1} box brings the 16-byte row holding each wanted entry. Per CTA: one
// producer warp issues the gathers for a tile of 1024 columns (each lane 4
// columns per instruction, 8 instructions per lane) into one of S stages
// (mbarrier full/empty pairs); the consumer warps sum the wanted halves.
// The LDG form (same sum) runs beside it for the ratio.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 gather4_probe.cu -o gather4_probe -lcuda
//
// Measured on one B200 (round 2; both sums checked equal, integer-valued x):
//   x          LDG (ILP 16)          TMA gather4 (1 CTA/SM)   (2 CTA/SM)
//   8 MB       79.7 us  210.6 G/s    989 us   17.0 G/s       1032 us  16.3 G/s
//   32 MB      96.9 us  173.2 G/s    1235 us  13.6 G/s       1235 us  13.6 G/s
//   512 MB     303 us    55.4 G/s    1260 us  13.3 G/s       1259 us  13.3 G/s
// The tensor-map gather retires about one 4-row gather4 per ~68 SM cycles
// (16-byte rows), independent of the CTAs per SM — the SM's TMA unit, not the
// L1->XBAR request path, is the limiter, and it is ~12x slower than LDG for
// scattered 8-byte entries. Verdict: no gather path through TMA for SpMV's
// random columns; the LDG gather ceiling stands.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>

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
__device__ __forceinline__ void gather4(void* dst, const CUtensorMap* tm, int c0, int r0, int r1, int r2, int r3,
                                        uint64_t* bar) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 ::"r"(smem_u32(dst)), "l"(tm), "r"(c0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(smem_u32(bar))
                 : "memory");
}

constexpr int TILE = 1024;   // columns per stage
constexpr int S = 6;         // stages
// a tensor copy's shared-memory destination must be 128-byte aligned: each
// gather4 (4 rows x 16 B = 64 B) gets its own 128-byte slot
constexpr int SLOT2 = 8;     // double2 per gather4 slot
constexpr int NCW = 4;       // consumer warps

__device__ __forceinline__ void warp_add(double* out, double acc) {   // one atomic per warp
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if ((threadIdx.x & 31) == 0) atomicAdd(out, acc);
}

__global__ void __launch_bounds__(32 * (NCW + 1), 1) g4_kernel(int64_t n, const int* __restrict__ idx,
                                                               const __grid_constant__ CUtensorMap tm,
                                                               double* __restrict__ out) {
    extern __shared__ __align__(128) double2 buf[];   // [S][TILE / 4 slots][SLOT2]
    __shared__ __align__(8) uint64_t full[S], empty[S];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t ntile = (n + TILE - 1) / TILE;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], NCW); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    int k = 0;
    if (warp == 0) {   // producer
        for (int64_t t = blockIdx.x; t < ntile; t += gridDim.x, ++k) {
            const int s = k % S;
            if (k >= S) mbar_wait(&empty[s], (uint32_t)((k / S) - 1) & 1u);
            if (lane == 0) mbar_expect(&full[s], TILE * 16);
            __syncwarp();
            const int64_t c0 = t * TILE;
#pragma unroll
            for (int r = 0; r < TILE / 128; ++r) {
                const int64_t i = c0 + r * 128 + lane * 4;
                int4 c = make_int4(0, 0, 0, 0);
                if (i + 3 < n) c = __ldg(reinterpret_cast<const int4*>(idx + i));   // tail: n is a multiple of TILE here
                gather4(&buf[(s * (TILE / 4) + r * 32 + lane) * SLOT2], &tm, 0, c.x >> 1, c.y >> 1, c.z >> 1, c.w >> 1,
                        &full[s]);
            }
        }
    } else {           // consumers
        double acc = 0;
        const int ct = threadIdx.x - 32;
        for (int64_t t = blockIdx.x; t < ntile; t += gridDim.x, ++k) {
            const int s = k % S;
            mbar_wait(&full[s], (uint32_t)(k / S) & 1u);
            const int64_t c0 = t * TILE;
            for (int i = ct; i < TILE; i += 32 * NCW) {
                const int c = __ldg(idx + c0 + i);
                const double2 v = buf[(s * (TILE / 4) + (i >> 2)) * SLOT2 + (i & 3)];
                acc += (c & 1) ? v.y : v.x;
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
        }
        warp_add(out, acc);
    }
}

__global__ void __launch_bounds__(256) ldg_kernel(int64_t n, const int* __restrict__ idx, const double* __restrict__ x,
                                                  double* __restrict__ out) {
    double acc = 0;
    constexpr int ILP = 16;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x * ILP;
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < n; b += stride) {
        int c[ILP];
#pragma unroll
        for (int u = 0; u < ILP; ++u) {
            const int64_t i = b + (int64_t)u * gridDim.x * blockDim.x;
            c[u] = i < n ? __ldg(idx + i) : 0;
        }
#pragma unroll
        for (int u = 0; u < ILP; ++u) {
            const int64_t i = b + (int64_t)u * gridDim.x * blockDim.x;
            acc += i < n ? __ldg(x + c[u]) : 0.0;
        }
    }
    warp_add(out, acc);
}

__global__ void iota(int64_t n, double* x) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] = (double)(i & 1023);
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    setvbuf(stdout, nullptr, _IONBF, 0);
    cudaFree(0);
    EncodeFn encode = cuTensorMapEncodeTiled;   // linked: -lcuda
    const int64_t n = 16LL << 20;   // config 2's nnz
    const size_t smem = (size_t)S * (TILE / 4) * SLOT2 * 16;
    cudaFuncSetAttribute(g4_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    for (int64_t xs : {1LL << 20, 4LL << 20, 64LL << 20}) {
        std::vector<int> h(n);
        std::mt19937_64 g(7);
        for (auto& v : h) v = (int)(g() % xs);
        int* idx;
        double *x, *out;
        cudaMalloc(&idx, n * 4);
        cudaMalloc(&x, xs * 8);
        cudaMalloc(&out, 8);
        cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice);
        iota<<<1024, 256>>>(xs, x);   // integer-valued: the two sums agree exactly in any order
        CUtensorMap tm;
        const cuuint64_t dims[2] = {2, (cuuint64_t)(xs / 2)};
        const cuuint64_t strides[1] = {16};
        const cuuint32_t box[2] = {2, 1};
        const cuuint32_t estr[2] = {1, 1};
        CUresult r = encode(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, x, dims, strides, box, estr,
                            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) { printf("encode failed %d\n", (int)r); return 1; }
        {
            double s1 = 0, s2 = 0;
            cudaMemset(out, 0, 8);
            ldg_kernel<<<sms * 8, 256>>>(n, idx, x, out);
            cudaMemcpy(&s1, out, 8, cudaMemcpyDeviceToHost);
            cudaMemset(out, 0, 8);
            g4_kernel<<<sms, 32 * (NCW + 1), smem>>>(n, idx, tm, out);
            cudaError_t e = cudaMemcpy(&s2, out, 8, cudaMemcpyDeviceToHost);
            printf("  check: LDG sum %.0f, gather4 sum %.0f (%s)%s\n", s1, s2, s1 == s2 ? "equal" : "DIFFER",
                   e == cudaSuccess ? "" : cudaGetErrorString(e));
            if (e != cudaSuccess || s1 != s2) return 1;
        }
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        printf("x = %lld doubles (%lld MB), %lld gathers\n", (long long)xs, (long long)(xs * 8 >> 20), (long long)n);
        for (int grid_mult : {1, 2}) {
            const int grid = sms * grid_mult;
            ldg_kernel<<<sms * 8, 256>>>(n, idx, x, out);
            cudaEventRecord(a);
            for (int rep = 0; rep < 5; ++rep) ldg_kernel<<<sms * 8, 256>>>(n, idx, x, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            double t = ms / 5 * 1e-3;
            if (grid_mult == 1)
                printf("  LDG (ILP 16)              : %8.1f us  %6.1f G gathers/s\n", t * 1e6, n / t / 1e9);
            g4_kernel<<<grid, 32 * (NCW + 1), smem>>>(n, idx, tm, out);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) { printf("g4 failed: %s\n", cudaGetErrorString(e)); return 1; }
            cudaEventRecord(a);
            for (int rep = 0; rep < 5; ++rep) g4_kernel<<<grid, 32 * (NCW + 1), smem>>>(n, idx, tm, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            t = ms / 5 * 1e-3;
            printf("  TMA gather4 (%d CTA/SM, S=%d): %8.1f us  %6.1f G gathers/s\n", grid_mult, S, t * 1e6, n / t / 1e9);
        }
        cudaFree(idx);
        cudaFree(x);
        cudaFree(out);
    }
    return 0;
}
