// sell_probe.cu — standalone experiment (not part of the library): SELL-32
// kernel refinements on the config-4 Laplacian (8192², uniform chunks of
// length 5, boundary chunks masked).
//   v0: library design (one chunk per warp, exact-size batch)
//   v1: v0 + the next chunk's metadata prefetched during the current one
//   v2: v1 + two chunks per warp when both are uniform with equal length
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ uint64_t pol_ef() { uint64_t p; asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ double ldd(const double* p, uint64_t pol) { double r; asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(r) : "l"(p), "l"(pol)); return r; }
__device__ __forceinline__ int ldi(const int* p, uint64_t pol) { int r; asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol)); return r; }

template <int N>
__device__ __forceinline__ double slots(const double* __restrict__ val, const int* __restrict__ col, const double* __restrict__ x,
                                        int64_t base, int j0, int len, double acc, uint64_t pol) {
    double v[N], xv[N]; int c[N];
#pragma unroll
    for (int u = 0; u < N; ++u) c[u] = ldi(col + base + (int64_t)(j0 + u) * 32, pol);
#pragma unroll
    for (int u = 0; u < N; ++u) v[u] = ldd(val + base + (int64_t)(j0 + u) * 32, pol);
#pragma unroll
    for (int u = 0; u < N; ++u) xv[u] = __ldg(x + c[u]);
#pragma unroll
    for (int u = 0; u < N; ++u) if (j0 + u < len) acc = fma(v[u], xv[u], acc);
    return acc;
}

template <int N>
__device__ __forceinline__ void slots2(const double* __restrict__ val, const int* __restrict__ col, const double* __restrict__ x,
                                       int64_t b0, int64_t b1, double& a0, double& a1, uint64_t pol) {
    double v0[N], v1[N], x0[N], x1[N]; int c0[N], c1[N];
#pragma unroll
    for (int u = 0; u < N; ++u) { c0[u] = ldi(col + b0 + u * 32, pol); c1[u] = ldi(col + b1 + u * 32, pol); }
#pragma unroll
    for (int u = 0; u < N; ++u) { v0[u] = ldd(val + b0 + u * 32, pol); v1[u] = ldd(val + b1 + u * 32, pol); }
#pragma unroll
    for (int u = 0; u < N; ++u) { x0[u] = __ldg(x + c0[u]); x1[u] = __ldg(x + c1[u]); }
#pragma unroll
    for (int u = 0; u < N; ++u) { a0 = fma(v0[u], x0[u], a0); a1 = fma(v1[u], x1[u], a1); }
}

__device__ __forceinline__ double chunk(const double* val, const int* col, const double* x, int64_t base, int clen, int len, uint64_t pol) {
    double acc = 0; int j = 0;
    for (; j + 8 <= clen; j += 8) acc = slots<8>(val, col, x, base, j, len, acc, pol);
    switch (clen - j) {
    case 1: acc = slots<1>(val, col, x, base, j, len, acc, pol); break;
    case 2: acc = slots<2>(val, col, x, base, j, len, acc, pol); break;
    case 3: acc = slots<3>(val, col, x, base, j, len, acc, pol); break;
    case 4: acc = slots<4>(val, col, x, base, j, len, acc, pol); break;
    case 5: acc = slots<5>(val, col, x, base, j, len, acc, pol); break;
    case 6: acc = slots<6>(val, col, x, base, j, len, acc, pol); break;
    case 7: acc = slots<7>(val, col, x, base, j, len, acc, pol); break;
    default: break;
    }
    return acc;
}

template <int V>
__global__ void __launch_bounds__(256) sell(int nrows, int nchunks, const int64_t* __restrict__ cptr, const int* __restrict__ clen_,
                                            const int* __restrict__ rowlen, const int* __restrict__ col, const double* __restrict__ val,
                                            const double* __restrict__ x, double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int warp = (blockIdx.x * 256 + threadIdx.x) >> 5;
    const int nw = (gridDim.x * 256) >> 5;
    const uint64_t pol = pol_ef();
    if (V == 0) {
        for (int c = warp; c < nchunks; c += nw) {
            const int cl = __ldg(clen_ + c);
            const int64_t base = __ldg(cptr + c) + lane;
            const int r = c * 32 + lane;
            const int cl2 = cl >= 0 ? cl : -cl;
            const int len = cl >= 0 ? cl : (r < nrows ? __ldg(rowlen + r) : 0);
            double acc = chunk(val, col, x, base, cl2, len, pol);
            if (r < nrows) y[r] = acc;
        }
    } else if (V == 1) {
        int c = warp;
        int cl = c < nchunks ? __ldg(clen_ + c) : 0;
        int64_t cp = c < nchunks ? __ldg(cptr + c) : 0;
        for (; c < nchunks; c += nw) {
            const int cn = c + nw;
            int cln = 0; int64_t cpn = 0;
            if (cn < nchunks) { cln = __ldg(clen_ + cn); cpn = __ldg(cptr + cn); }
            const int r = c * 32 + lane;
            const int cl2 = cl >= 0 ? cl : -cl;
            const int len = cl >= 0 ? cl : (r < nrows ? __ldg(rowlen + r) : 0);
            double acc = chunk(val, col, x, cp + lane, cl2, len, pol);
            if (r < nrows) y[r] = acc;
            cl = cln; cp = cpn;
        }
    } else {
        // two chunks (c, c + nw) per iteration
        for (int c = warp; c < nchunks; c += 2 * nw) {
            const int d = c + nw;
            const int cl0 = __ldg(clen_ + c);
            const int cl1 = d < nchunks ? __ldg(clen_ + d) : -1;
            const int64_t b0 = __ldg(cptr + c) + lane;
            const int64_t b1 = d < nchunks ? __ldg(cptr + d) + lane : 0;
            const int r0 = c * 32 + lane, r1 = d * 32 + lane;
            double a0 = 0, a1 = 0;
            if (cl0 == cl1 && cl0 == 5) {
                slots2<5>(val, col, x, b0, b1, a0, a1, pol);
            } else {
                const int l0 = cl0 >= 0 ? cl0 : (r0 < nrows ? __ldg(rowlen + r0) : 0);
                a0 = chunk(val, col, x, b0, cl0 >= 0 ? cl0 : -cl0, l0, pol);
                if (d < nchunks) {
                    const int l1 = cl1 >= 0 ? cl1 : (r1 < nrows ? __ldg(rowlen + r1) : 0);
                    a1 = chunk(val, col, x, b1, cl1 >= 0 ? cl1 : -cl1, l1, pol);
                }
            }
            if (r0 < nrows) y[r0] = a0;
            if (d < nchunks && r1 < nrows) y[r1] = a1;
        }
    }
}

// v3: v1 + the next chunk's 5 column and value slots loaded before the
// current chunk's x gathers (uniform length-5 chunks; others fall back)
__global__ void __launch_bounds__(256) sell_v3(int nrows, int nchunks, const int64_t* __restrict__ cptr, const int* __restrict__ clen_,
                                               const int* __restrict__ rowlen, const int* __restrict__ col, const double* __restrict__ val,
                                               const double* __restrict__ x, double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int warp = (blockIdx.x * 256 + threadIdx.x) >> 5;
    const int nw = (gridDim.x * 256) >> 5;
    const uint64_t pol = pol_ef();
    int c = warp;
    if (c >= nchunks) return;
    int cl = __ldg(clen_ + c);
    int64_t cp = __ldg(cptr + c);
    int ci[5]; double cv[5];
    if (cl == 5) {
#pragma unroll
        for (int u = 0; u < 5; ++u) { ci[u] = ldi(col + cp + lane + u * 32, pol); cv[u] = ldd(val + cp + lane + u * 32, pol); }
    }
    for (; c < nchunks; c += nw) {
        const int cn = c + nw;
        int cln = 0; int64_t cpn = 0;
        if (cn < nchunks) { cln = __ldg(clen_ + cn); cpn = __ldg(cptr + cn); }
        const int r = c * 32 + lane;
        double acc = 0;
        if (cl == 5) {
            double xv[5];
#pragma unroll
            for (int u = 0; u < 5; ++u) xv[u] = __ldg(x + ci[u]);
            double v[5];
#pragma unroll
            for (int u = 0; u < 5; ++u) v[u] = cv[u];
            if (cln == 5) {
#pragma unroll
                for (int u = 0; u < 5; ++u) { ci[u] = ldi(col + cpn + lane + u * 32, pol); cv[u] = ldd(val + cpn + lane + u * 32, pol); }
            }
#pragma unroll
            for (int u = 0; u < 5; ++u) acc = fma(v[u], xv[u], acc);
        } else {
            const int cl2 = cl >= 0 ? cl : -cl;
            const int len = cl >= 0 ? cl : (r < nrows ? __ldg(rowlen + r) : 0);
            acc = chunk(val, col, x, cp + lane, cl2, len, pol);
            if (cln == 5) {
#pragma unroll
                for (int u = 0; u < 5; ++u) { ci[u] = ldi(col + cpn + lane + u * 32, pol); cv[u] = ldd(val + cpn + lane + u * 32, pol); }
            }
        }
        if (r < nrows) y[r] = acc;
        cl = cln; cp = cpn;
    }
}

template <int V>
void run(const char* name, int grid, int nrows, int nchunks, const int64_t* cp, const int* cl, const int* rl, const int* col,
         const double* val, const double* x, double* y) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    sell<V><<<grid, 256>>>(nrows, nchunks, cp, cl, rl, col, val, x, y);
    cudaEventRecord(a);
    for (int i = 0; i < 10; ++i) sell<V><<<grid, 256>>>(nrows, nchunks, cp, cl, rl, col, val, x, y);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    const double bytes = 5368315908.0;
    printf("%-28s grid=%6d  %.1f us  %.0f GB/s algorithmic\n", name, grid, ms * 100, bytes / (ms / 10 * 1e-3) / 1e9);
}

int main() {
    const int n = 8192; const int64_t R = (int64_t)n * n;
    const int nchunks = (int)(R / 32);
    std::vector<int> clen(nchunks), rowlen(R);
    std::vector<int64_t> cptr(nchunks + 1);
    int64_t slots = 0;
    for (int c = 0; c < nchunks; ++c) {
        int mx = 0, mn = 99;
        for (int l = 0; l < 32; ++l) {
            int64_t i = (int64_t)c * 32 + l; int64_t r = i / n, cc = i % n;
            int len = 1 + (r > 0) + (r < n - 1) + (cc > 0) + (cc < n - 1);
            rowlen[i] = len; mx = len > mx ? len : mx; mn = len < mn ? len : mn;
        }
        clen[c] = mn == mx ? mx : -mx;
        cptr[c] = slots; slots += (int64_t)mx * 32;
    }
    cptr[nchunks] = slots;
    std::vector<int> col(slots, 0);
    std::vector<double> val(slots, 0.0);
    for (int c = 0; c < nchunks; ++c)
        for (int l = 0; l < 32; ++l) {
            int64_t i = (int64_t)c * 32 + l; int64_t r = i / n, cc = i % n; int j = 0;
            auto put = [&](int64_t cix, double v) { col[cptr[c] + j * 32 + l] = (int)cix; val[cptr[c] + j * 32 + l] = v; ++j; };
            if (r > 0) put(i - n, -1); if (cc > 0) put(i - 1, -1); put(i, 4); if (cc < n - 1) put(i + 1, -1); if (r < n - 1) put(i + n, -1);
        }
    int64_t *dcp; int *dcl, *drl, *dcol; double *dval, *dx, *dy;
    CK(cudaMalloc(&dcp, 8 * (nchunks + 1))); CK(cudaMalloc(&dcl, 4 * nchunks)); CK(cudaMalloc(&drl, 4 * R));
    CK(cudaMalloc(&dcol, 4 * slots)); CK(cudaMalloc(&dval, 8 * slots)); CK(cudaMalloc(&dx, 8 * R)); CK(cudaMalloc(&dy, 8 * R));
    CK(cudaMemcpy(dcp, cptr.data(), 8 * (nchunks + 1), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dcl, clen.data(), 4 * nchunks, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(drl, rowlen.data(), 4 * R, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dcol, col.data(), 4 * slots, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dval, val.data(), 8 * slots, cudaMemcpyHostToDevice));
    CK(cudaMemset(dx, 0, 8 * R));
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int g : {sms * 8, sms * 4, sms * 6}) {
        run<1>("v1 + meta prefetch", g, (int)R, nchunks, dcp, dcl, drl, dcol, dval, dx, dy);
        cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
        sell_v3<<<g, 256>>>((int)R, nchunks, dcp, dcl, drl, dcol, dval, dx, dy);
        cudaEventRecord(a);
        for (int i = 0; i < 10; ++i) sell_v3<<<g, 256>>>((int)R, nchunks, dcp, dcl, drl, dcol, dval, dx, dy);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        printf("%-28s grid=%6d  %.1f us  %.0f GB/s algorithmic\n", "v3 + slot prefetch", g, ms * 100, 5368315908.0 / (ms / 10 * 1e-3) / 1e9);
    }
    CK(cudaDeviceSynchronize());
    return 0;
}
