/*
 * oracle.c — TEST INFRASTRUCTURE ONLY. The plain, slow, obviously correct CPU
 * definition of what the SpMV hot path computes.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library. It shares no code, header or
 * helper with the CUDA path (paper_conf_sc_dastgeerlk12_b200/csrc), and the
 * CUDA path never calls it.
 *
 * Paper: U. Dastgeer, L. Li, C. Kessler, "The PEPPHER Composition Tool",
 * MuCoCoS/SC 2012. Citations P@N = byte offset N in /root/reference/PAPER.md
 * (one physical line).
 *
 *  - The operation: the component `spmv(values, nnz, nrows, ncols, first,
 *    colidxs, rowPtr, x, y)` of §V-A (P@32944 + P@31037, garble G1), y = A·x
 *    over CSR. Reading A1: row i's entries are positions
 *    [rowPtr[i]-first, rowPtr[i+1]-first) of values/colidxs. A4: y is
 *    written, not accumulated. A6: empty rows give +0.0. A8: duplicate
 *    columns are summed, order of columns is irrelevant.
 *  - The "one serial C++ implementation for the CPU" variant (P@33595) is
 *    oracle_spmv_seq: ascending k, accumulator +0.0, product rounded then sum
 *    rounded (compiled with -ffp-contract=off, SSE2 doubles: no FMA, no x87).
 *  - Partitioned calls produce the "concatenation of intermediate output
 *    results produced by each sub-task" (§IV-F, P@27875): oracle_spmv_seq on
 *    a row block with its own `first` is exactly that sub-task.
 *  - oracle_spmv_rows_parallel: the same loop with rows split over OpenMP
 *    threads; each row's sum order is unchanged, so it is bitwise equal to
 *    oracle_spmv_seq (used as the timing baseline and for large sizes).
 *  - oracle_abs_rowsum: S_i = Σ_k |a_ik|·|x_col| for the per-row error bound
 *    |y - y_ref| <= 2·nnz_row·2^-52·S_i stated in BASELINE.json north_star.
 *  - oracle_partition_nnz: the nnz-balanced contiguous row-block rule of
 *    DESIGN.md reading A9 (P@27578 "partitioning and dividing the work into
 *    several chunks"), written as a linear scan of its definition.
 *
 * Build: gcc -O2 -ffp-contract=off -fno-fast-math -fopenmp -shared -fPIC
 */
#include <stdint.h>
#include <math.h>

#define ORACLE_EXPORT __attribute__((visibility("default")))

/* y[i] = sum_{k=row_ptr[i]-first}^{row_ptr[i+1]-first-1} val[k] * x[col[k]], i in [0,nrows) */
ORACLE_EXPORT void oracle_spmv_seq(int64_t nrows, int64_t first, const int64_t* row_ptr,
                                   const int32_t* col, const double* val,
                                   const double* x, double* y) {
    for (int64_t i = 0; i < nrows; ++i) {
        double acc = +0.0;
        for (int64_t k = row_ptr[i] - first; k < row_ptr[i + 1] - first; ++k) {
            double prod = val[k] * x[col[k]];
            acc = acc + prod;
        }
        y[i] = acc;
    }
}

/* same definition, rows distributed over threads (row sums unchanged) */
ORACLE_EXPORT void oracle_spmv_rows_parallel(int64_t nrows, int64_t first, const int64_t* row_ptr,
                                             const int32_t* col, const double* val,
                                             const double* x, double* y) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < nrows; ++i) {
        double acc = +0.0;
        for (int64_t k = row_ptr[i] - first; k < row_ptr[i + 1] - first; ++k) {
            double prod = val[k] * x[col[k]];
            acc = acc + prod;
        }
        y[i] = acc;
    }
}

/* one row i (for sampled parity at full sizes) */
ORACLE_EXPORT double oracle_spmv_row(int64_t i, int64_t first, const int64_t* row_ptr,
                                     const int32_t* col, const double* val, const double* x) {
    double acc = +0.0;
    for (int64_t k = row_ptr[i] - first; k < row_ptr[i + 1] - first; ++k) {
        double prod = val[k] * x[col[k]];
        acc = acc + prod;
    }
    return acc;
}

/* ---- fp32 instance: the paper's own `float` signature (P@32944), SURVEY
   §8(f) f3. Same definition with float values, float x and a float
   accumulator: product rounded to float, then sum rounded to float,
   ascending k (SSE single precision, no FMA: -ffp-contract=off). */
ORACLE_EXPORT void oracle_spmv_seq_f32(int64_t nrows, int64_t first, const int64_t* row_ptr,
                                       const int32_t* col, const float* val, const float* x, float* y) {
    for (int64_t i = 0; i < nrows; ++i) {
        float acc = +0.0f;
        for (int64_t k = row_ptr[i] - first; k < row_ptr[i + 1] - first; ++k) {
            float prod = val[k] * x[col[k]];
            acc = acc + prod;
        }
        y[i] = acc;
    }
}

ORACLE_EXPORT void oracle_spmv_rows_parallel_f32(int64_t nrows, int64_t first, const int64_t* row_ptr,
                                                 const int32_t* col, const float* val, const float* x, float* y) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < nrows; ++i) {
        float acc = +0.0f;
        for (int64_t k = row_ptr[i] - first; k < row_ptr[i + 1] - first; ++k) {
            float prod = val[k] * x[col[k]];
            acc = acc + prod;
        }
        y[i] = acc;
    }
}

/* S_i = sum |a| |x| of an fp32 matrix, accumulated in double (bound only) */
ORACLE_EXPORT void oracle_abs_rowsum_f32(int64_t nrows, int64_t first, const int64_t* row_ptr,
                                         const int32_t* col, const float* val, const float* x, double* s) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < nrows; ++i) {
        double acc = 0.0;
        for (int64_t k = row_ptr[i] - first; k < row_ptr[i + 1] - first; ++k)
            acc = acc + fabs((double)val[k]) * fabs((double)x[col[k]]);
        s[i] = acc;
    }
}

/* S_i for one row i (sampled bound checks at full size) */
ORACLE_EXPORT double oracle_abs_row(int64_t i, int64_t first, const int64_t* row_ptr,
                                    const int32_t* col, const double* val, const double* x) {
    double acc = 0.0;
    for (int64_t k = row_ptr[i] - first; k < row_ptr[i + 1] - first; ++k)
        acc = acc + fabs(val[k]) * fabs(x[col[k]]);
    return acc;
}

/* S_i = sum |a_ik| |x_col|  (bound ingredient, P6) */
ORACLE_EXPORT void oracle_abs_rowsum(int64_t nrows, int64_t first, const int64_t* row_ptr,
                                     const int32_t* col, const double* val,
                                     const double* x, double* s) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < nrows; ++i) {
        double acc = 0.0;
        for (int64_t k = row_ptr[i] - first; k < row_ptr[i + 1] - first; ++k)
            acc = acc + fabs(val[k]) * fabs(x[col[k]]);
        s[i] = acc;
    }
}

/* Iterated SpMV x_{k+1} = A x_k, K times, square A (reading A11).  x is
   overwritten with x_K; tmp has nrows entries.  If z != NULL it is iterated
   alongside as z_{k+1} = |A| z_k from z_0 = |x_0| (bound vector of P7). */
ORACLE_EXPORT void oracle_spmv_iterate(int64_t K, int64_t nrows, int64_t first, const int64_t* row_ptr,
                                       const int32_t* col, const double* val,
                                       double* x, double* tmp, double* z, double* ztmp) {
    if (z) for (int64_t i = 0; i < nrows; ++i) z[i] = fabs(x[i]);
    for (int64_t it = 0; it < K; ++it) {
        oracle_spmv_rows_parallel(nrows, first, row_ptr, col, val, x, tmp);
        for (int64_t i = 0; i < nrows; ++i) x[i] = tmp[i];
        if (z) {
            oracle_abs_rowsum(nrows, first, row_ptr, col, val, z, ztmp);
            for (int64_t i = 0; i < nrows; ++i) z[i] = ztmp[i];
        }
    }
}

/* nnz-balanced contiguous row blocks (A9):
   bounds[p] = min { r in [0,nrows] : row_ptr[r] - first >= ceil(p*nnz/P) },
   bounds[0] = 0, bounds[P] = nrows. Linear scan of the definition. */
ORACLE_EXPORT void oracle_partition_nnz(int64_t nrows, int64_t first, const int64_t* row_ptr,
                                        int64_t P, int64_t* bounds) {
    int64_t nnz = row_ptr[nrows] - first;
    bounds[0] = 0;
    for (int64_t p = 1; p < P; ++p) {
        /* ceil(p*nnz/P) without overflow for nnz < 2^62/P */
        int64_t target = (p * nnz + P - 1) / P;
        int64_t r = 0;
        while (r < nrows && row_ptr[r] - first < target) ++r;
        bounds[p] = r;
    }
    bounds[P] = nrows;
}
