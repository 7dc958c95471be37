/*
 * ORACLE -- TEST INFRASTRUCTURE ONLY (cpu_baseline leg of bench.py).
 * Only tests/ and bench.py may load this code; the product never does and
 * shares no code with it.
 *
 * What it computes: the same definition as coo_spmv.c,
 *
 *     y[r] = beta*y0[r] + alpha * sum_{(r,c,v) in COO} v * x[c]
 *
 * (BASELINE.json north_star alpha/beta form),
 * but accumulated in the matrix's own precision -- the plain COO loop a CPU
 * user would run, which SURVEY.md §8(d) and BASELINE.md §4 name as the
 * timed CPU baseline (the long-double coo_spmv.c stays the checker). It is
 * the paper's CPU comparison point in spirit (multi-threaded CSR SpMV on the
 * host, Table VI), not MKL.
 *
 * The COO must be sorted by row (any column order). With nthreads > 1 the
 * entries are cut into nthreads contiguous ranges at row boundaries
 * (OpenMP, one range per thread); each row is summed by one thread in the
 * given entry order, so the result does not depend on the thread count.
 * Rows without entries get y = beta*y0 (beta == 0: 0; y0 not read).
 *
 * Pinned by tests/test_oracle_pins.py: within the recursive-summation bound
 * of the long-double definition, and bit-identical across thread counts.
 */
#include <stdint.h>
#include <stdlib.h>
#include <omp.h>

#define DEFINE_NATIVE(NAME, T)                                                                              \
    int NAME(int64_t nrows, int64_t nnz, const int64_t *row, const int64_t *col, const T *val, T alpha,     \
             const T *x, T beta, const T *y0, T *y, int nthreads) {                                         \
        for (int64_t e = 1; e < nnz; ++e)                                                                   \
            if (row[e] < row[e - 1]) return 1; /* not row-sorted */                                         \
        if (nthreads < 1) nthreads = 1;                                                                     \
        _Pragma("omp parallel num_threads(nthreads)")                                                       \
        {                                                                                                   \
            const int t = omp_get_thread_num(), nt = omp_get_num_threads();                                 \
            /* my rows: [r0, r1), cut so every thread gets ~nnz/nt entries */                              \
            int64_t e0 = nnz * t / nt, e1 = nnz * (t + 1) / nt;                                             \
            int64_t r0 = (t == 0) ? 0 : (e0 < nnz ? row[e0] : nrows);                                       \
            int64_t r1 = (t == nt - 1) ? nrows : (e1 < nnz ? row[e1] : nrows);                              \
            if (t > 0 && e0 > 0 && e0 < nnz && row[e0 - 1] == row[e0]) r0 = row[e0] + 1;                    \
            if (t < nt - 1 && e1 > 0 && e1 < nnz && row[e1 - 1] == row[e1]) r1 = row[e1] + 1;                \
            if (r1 < r0) r1 = r0;                                                                           \
            /* first entry of row r0 */                                                                     \
            int64_t lo = 0, hi = nnz;                                                                       \
            while (lo < hi) {                                                                               \
                const int64_t mid = lo + (hi - lo) / 2;                                                     \
                if (row[mid] < r0) lo = mid + 1; else hi = mid;                                             \
            }                                                                                               \
            int64_t e = lo;                                                                                 \
            for (int64_t r = r0; r < r1; ++r) {                                                             \
                T acc = (T)0;                                                                               \
                for (; e < nnz && row[e] == r; ++e) acc += val[e] * x[col[e]];                              \
                y[r] = (beta != (T)0) ? alpha * acc + beta * y0[r] : alpha * acc;                           \
            }                                                                                               \
        }                                                                                                   \
        return 0;                                                                                           \
    }

DEFINE_NATIVE(oracle_coo_native_f64, double)
DEFINE_NATIVE(oracle_coo_native_f32, float)
