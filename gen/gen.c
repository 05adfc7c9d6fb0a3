/*
 * gen.c — seeded synthetic CSR inputs for the SpMV hot path.
 *
 * This module holds NONE of the method's arithmetic (no products, no sums of
 * matrix entries). It only produces structure (row_ptr, col_idx), values and
 * dense vectors from a counter-based generator, so that both the oracle
 * (oracle/) and the CUDA path (paper_conf_sc_dastgeerlk12_b200/) can be fed
 * the same inputs without sharing any code with each other.
 *
 * Workload recipes follow SURVEY.md §8(d) and DESIGN.md §"Input recipe":
 *   - 2D 5-point Laplacian, Dirichlet, row-major grid, +4 diagonal, -1 off
 *     (SURVEY §8(c) reading A12; configs 1 and 4 of BASELINE.json);
 *   - uniform random, exactly k distinct sorted columns per row (config 2);
 *   - power-law row lengths P(len=k) ∝ k^-alpha on [1,kmax] (A13, config 3);
 *   - banded, half-bandwidth b (A15, config 5);
 *   - permutation / diagonal (oracle pins P2/P3).
 *
 * Random numbers: gen_u64(seed, a, b) = SplitMix64 finaliser chain over
 * (seed, a, b); a pure function of its three counters, so any slice of a
 * matrix (one rank's row block) is reproducible independently.
 *
 * Build: gcc -O2 -fopenmp -shared -fPIC gen.c -o libpepp_gen.so
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define GEN_EXPORT __attribute__((visibility("default")))

static inline uint64_t sm64(uint64_t z) {
    z += 0x9e3779b97f4a7c15ULL;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}

GEN_EXPORT uint64_t gen_u64(uint64_t seed, uint64_t a, uint64_t b) {
    return sm64(sm64(sm64(seed) ^ a) ^ (b * 0xd1b54a32d192ed03ULL));
}

/* uniform in [0,1) with 53 random bits */
static inline double u01(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }

/* ------------------------------------------------------------------ */
/* value / vector modes                                                */
/*   0: real  U[-1,1)  (multiples of 2^-52)                            */
/*   1: int   {±1,±2,±3,±4}                                            */
/*   2: int   uniform in [-8,8]                                        */
/*   3: ones                                                            */
/*   4: real  U[-1,1) but never exactly 0                               */
/* ------------------------------------------------------------------ */
static inline double draw_value(int mode, uint64_t r) {
    switch (mode) {
    case 0: return 2.0 * u01(r) - 1.0;
    case 1: { double m = (double)((r >> 1) % 4 + 1); return (r & 1) ? -m : m; }
    case 2: return (double)((int64_t)((r >> 8) % 17) - 8);
    case 3: return 1.0;
    case 4: { double v = 2.0 * u01(r) - 1.0; return v == 0.0 ? 0.5 : v; }
    default: return 0.0;
    }
}

/* out[i] = value(seed, offset + i) for i in [0,n); stream id 7 */
GEN_EXPORT void gen_values(uint64_t seed, int mode, int64_t offset, int64_t n, double* out) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i)
        out[i] = draw_value(mode, gen_u64(seed, 7, (uint64_t)(offset + i)));
}

/* ------------------------------------------------------------------ */
/* 2D 5-point Laplacian on an n x n grid (A12)                          */
/* row i = r*n + c; neighbours in ascending column order:               */
/*   (r-1,c) (r,c-1) (r,c) (r,c+1) (r+1,c); absent ones dropped.         */
/* ------------------------------------------------------------------ */
static inline int lap_len(int64_t n, int64_t i) {
    int64_t r = i / n, c = i % n;
    return 1 + (r > 0) + (r < n - 1) + (c > 0) + (c < n - 1);
}

/* number of nonzeros in rows [0, i) — closed form, so slices need no scan */
static int64_t lap_prefix(int64_t n, int64_t i) {
    if (n == 1) return i;
    int64_t r = i / n, c = i % n;
    /* full grid rows before row r */
    int64_t full = 0;
    if (r > 0) {
        int64_t edge = 4 * n - 2;           /* nnz of first / last grid row */
        int64_t mid = 5 * n - 2;            /* nnz of an interior grid row */
        int64_t rmid = (r < n - 1 ? r : n - 1) - 1;   /* interior grid rows among [1, r) */
        full = edge + rmid * mid + (r == n ? edge : 0);
    }
    /* partial row r: columns [0, c) */
    int64_t part = 0;
    if (c > 0) {
        int vert = (r > 0) + (r < n - 1);   /* vertical neighbours per cell */
        /* cells: diagonal + vert each, plus horizontal: col 0 has 1, interior 2, col n-1 has 1 */
        int64_t horiz = (c >= 1 ? 1 : 0) + 2 * (c - 1 > 0 ? c - 1 : 0);
        /* horizontal neighbour count of cells 0..c-1: cell 0 -> 1 (right),
           cells 1..c-1 -> 2 each unless cell is n-1 (only when c == n, excluded) */
        part = c * (1 + vert) + horiz;
    }
    return full + part;
}

GEN_EXPORT int64_t gen_laplacian2d_nnz(int64_t n) { return lap_prefix(n, n * n); }

/* row_ptr[i - r0] = first + nnz(rows [r0, i)) for i in [r0, r1]  (global offsets if first=lap_prefix(r0)) */
GEN_EXPORT void gen_laplacian2d_rowptr(int64_t n, int64_t r0, int64_t r1, int64_t* row_ptr) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = r0; i <= r1; ++i) row_ptr[i - r0] = lap_prefix(n, i);
}

/* fill columns and values (+4 / -1) for rows [r0, r1); entries of row i go to
   col[row_ptr_global(i) - base] where base = lap_prefix(n, r0) */
GEN_EXPORT void gen_laplacian2d_fill(int64_t n, int64_t r0, int64_t r1, int32_t* col, double* val) {
    int64_t base = lap_prefix(n, r0);
    #pragma omp parallel for schedule(static)
    for (int64_t i = r0; i < r1; ++i) {
        int64_t k = lap_prefix(n, i) - base;
        int64_t r = i / n, c = i % n;
        if (r > 0)     { col[k] = (int32_t)(i - n); if (val) val[k] = -1.0; ++k; }
        if (c > 0)     { col[k] = (int32_t)(i - 1); if (val) val[k] = -1.0; ++k; }
        col[k] = (int32_t)i; if (val) val[k] = 4.0; ++k;
        if (c < n - 1) { col[k] = (int32_t)(i + 1); if (val) val[k] = -1.0; ++k; }
        if (r < n - 1) { col[k] = (int32_t)(i + n); if (val) val[k] = -1.0; ++k; }
    }
}

/* ------------------------------------------------------------------ */
/* row-length recipes -> lengths array len[i - r0] for rows [r0, r1)    */
/* ------------------------------------------------------------------ */
/* kind 0: constant k; kind 1: power law alpha, kmax (inverse CDF);      */
/* kind 2: banded half-bandwidth b on an nrows x nrows matrix            */
GEN_EXPORT void gen_row_lengths(int kind, uint64_t seed, int64_t nrows, int64_t ncols,
                                double alpha, int64_t kparam, int64_t r0, int64_t r1,
                                int32_t* len) {
    if (kind == 0) {
        int64_t k = kparam < ncols ? kparam : ncols;
        #pragma omp parallel for schedule(static)
        for (int64_t i = r0; i < r1; ++i) len[i - r0] = (int32_t)k;
    } else if (kind == 1) {
        int64_t kmax = kparam < ncols ? kparam : ncols;
        double* cdf = (double*)malloc(sizeof(double) * (size_t)(kmax + 1));
        double s = 0.0;
        cdf[0] = 0.0;
        for (int64_t k = 1; k <= kmax; ++k) { s += pow((double)k, -alpha); cdf[k] = s; }
        for (int64_t k = 1; k <= kmax; ++k) cdf[k] /= s;
        cdf[kmax] = 1.0;
        #pragma omp parallel for schedule(static)
        for (int64_t i = r0; i < r1; ++i) {
            double u = u01(gen_u64(seed, 11, (uint64_t)i));
            /* smallest k with cdf[k] > u */
            int64_t lo = 1, hi = kmax;
            while (lo < hi) { int64_t mid = (lo + hi) / 2; if (cdf[mid] > u) hi = mid; else lo = mid + 1; }
            len[i - r0] = (int32_t)lo;
        }
        free(cdf);
    } else {
        int64_t b = kparam;
        #pragma omp parallel for schedule(static)
        for (int64_t i = r0; i < r1; ++i) {
            int64_t lo = i - b < 0 ? 0 : i - b;
            int64_t hi = i + b > ncols - 1 ? ncols - 1 : i + b;
            len[i - r0] = (int32_t)(hi >= lo ? hi - lo + 1 : 0);
        }
    }
}

/* exclusive prefix sum of lengths into row_ptr (n+1 entries), starting at first */
GEN_EXPORT void gen_lengths_to_rowptr(int64_t n, const int32_t* len, int64_t first, int64_t* row_ptr) {
    int64_t s = first;
    for (int64_t i = 0; i < n; ++i) { row_ptr[i] = s; s += len[i]; }
    row_ptr[n] = s;
}

/* columns for banded rows [r0, r1): contiguous [i-b, i+b] ∩ [0, ncols) */
GEN_EXPORT void gen_banded_fill(int64_t ncols, int64_t b, int64_t r0, int64_t r1,
                                const int64_t* row_ptr, int32_t* col) {
    int64_t base = row_ptr[0];
    #pragma omp parallel for schedule(static)
    for (int64_t i = r0; i < r1; ++i) {
        int64_t k = row_ptr[i - r0] - base;
        int64_t lo = i - b < 0 ? 0 : i - b;
        int64_t hi = i + b > ncols - 1 ? ncols - 1 : i + b;
        for (int64_t c = lo; c <= hi; ++c) col[k++] = (int32_t)c;
    }
}

static int cmp_i32(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    return (x > y) - (x < y);
}

/* distinct uniform random columns per row (A16: sampling without replacement),
   stored sorted. Row i draws from gen_u64(seed, 13 + t, i) for t = 0,1,2,...
   Rejection sampling with a per-row open-addressing set; if len > ncols/2 the
   complement is sampled instead. */
GEN_EXPORT void gen_random_cols_fill(uint64_t seed, int64_t ncols, int64_t r0, int64_t r1,
                                     const int64_t* row_ptr, int32_t* col) {
    int64_t base = row_ptr[0];
    #pragma omp parallel
    {
        int64_t cap = 0;
        int64_t* table = NULL;
        #pragma omp for schedule(dynamic, 1024)
        for (int64_t i = r0; i < r1; ++i) {
            int64_t k0 = row_ptr[i - r0] - base;
            int64_t len = row_ptr[i - r0 + 1] - row_ptr[i - r0];
            if (len == 0) continue;
            int32_t* out = col + k0;
            int complement = (len > ncols / 2);
            int64_t want = complement ? ncols - len : len;
            int64_t need = 16;
            while (need < 2 * want + 2) need <<= 1;
            if (need > cap) { free(table); cap = need; table = (int64_t*)malloc(sizeof(int64_t) * cap); }
            for (int64_t t = 0; t < need; ++t) table[t] = -1;
            int64_t got = 0; uint64_t t = 0;
            int32_t* pick = complement ? (int32_t*)malloc(sizeof(int32_t) * (want + 1)) : out;
            while (got < want) {
                uint64_t r = gen_u64(seed, 13 + t, (uint64_t)i); ++t;
                int64_t c = (int64_t)(r % (uint64_t)ncols);
                uint64_t h = (uint64_t)c * 0x9e3779b97f4a7c15ULL;
                int64_t slot = (int64_t)(h >> 40) & (need - 1);
                int dup = 0;
                while (table[slot] != -1) { if (table[slot] == c) { dup = 1; break; } slot = (slot + 1) & (need - 1); }
                if (dup) continue;
                table[slot] = c;
                pick[got++] = (int32_t)c;
            }
            qsort(pick, (size_t)want, sizeof(int32_t), cmp_i32);
            if (complement) {
                int64_t p = 0, o = 0;
                for (int64_t c = 0; c < ncols; ++c) {
                    if (p < want && pick[p] == c) { ++p; continue; }
                    out[o++] = (int32_t)c;
                }
                free(pick);
            }
        }
        free(table);
    }
}

/* permutation pi of [0,n) by Fisher–Yates driven by gen_u64(seed, 17, j) */
GEN_EXPORT void gen_permutation(uint64_t seed, int64_t n, int32_t* perm) {
    for (int64_t i = 0; i < n; ++i) perm[i] = (int32_t)i;
    for (int64_t j = n - 1; j > 0; --j) {
        int64_t t = (int64_t)(gen_u64(seed, 17, (uint64_t)j) % (uint64_t)(j + 1));
        int32_t tmp = perm[j]; perm[j] = perm[t]; perm[t] = tmp;
    }
}
