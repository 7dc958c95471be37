/*
 * ORACLE -- TEST INFRASTRUCTURE ONLY.
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
 * --impl reference) may load this code. The product path (libcrsd.so and the
 * paper_conf_icpp_sunzwzyr11_b200 package) never calls it, and it shares no
 * code with the product.
 *
 * What it computes: the plain definition of the operation CRSD accelerates.
 * The paper's problem statement is SpMV y = A*x with y stored (PAPER.md
 * P:L33-39 abstract, "the result should be stored at ... y");
 * BASELINE.json north_star generalises it to y = alpha*A*x + beta*y. CRSD
 * reaches this exact result up to rounding order, so the
 * oracle is the definition written out:
 *
 *     y[r] = beta*y0[r] + alpha * sum_{(r,c,v) in COO} v * x[c]
 *
 * accumulated in long double (x87 80-bit) in the order the entries are given,
 * compiled with -ffp-contract=off. When beta == 0, y0 is not read (BLAS
 * convention; reading R7). It also emits the per-row scale
 *     scale[r] = |alpha| * sum |v|*|x[c]| + |beta|*|y0[r]|
 * that the parity criterion divides by (north_star: max|y-y_ref|/(|A||x|)_row).
 *
 * Pinned by tests/test_oracle_pins.py against a dense brute-force product,
 * scipy.sparse, and stencil closed forms.
 */
#include <stdint.h>
#include <stdlib.h>
#include <math.h>

#define ORACLE_OK 0
#define ORACLE_ERR_RANGE 1
#define ORACLE_ERR_ALLOC 2

static int check_range(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row, const int64_t *col) {
    for (int64_t e = 0; e < nnz; ++e)
        if (row[e] < 0 || row[e] >= nrows || col[e] < 0 || col[e] >= ncols) return ORACLE_ERR_RANGE;
    return ORACLE_OK;
}

int oracle_coo_spmv_f64(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row, const int64_t *col,
                        const double *val, double alpha, const double *x, double beta, const double *y0,
                        double *y_out, double *scale_out) {
    int rc = check_range(nrows, ncols, nnz, row, col);
    if (rc) return rc;
    long double *acc = (long double *)calloc((size_t)(nrows > 0 ? nrows : 1), sizeof(long double));
    long double *mag = (long double *)calloc((size_t)(nrows > 0 ? nrows : 1), sizeof(long double));
    if (!acc || !mag) { free(acc); free(mag); return ORACLE_ERR_ALLOC; }
    for (int64_t e = 0; e < nnz; ++e) {
        long double p = (long double)val[e] * (long double)x[col[e]];
        acc[row[e]] += p;
        mag[row[e]] += fabsl(p);
    }
    for (int64_t r = 0; r < nrows; ++r) {
        long double yr = (long double)alpha * acc[r];
        long double sr = fabsl((long double)alpha) * mag[r];
        if (beta != 0.0) {
            yr += (long double)beta * (long double)y0[r];
            sr += fabsl((long double)beta) * fabsl((long double)y0[r]);
        }
        y_out[r] = (double)yr;
        if (scale_out) scale_out[r] = (double)sr;
    }
    free(acc);
    free(mag);
    return ORACLE_OK;
}

/* Same definition for single precision inputs (taken exactly as given);
 * the result is returned in double so the comparison sees the oracle's
 * long-double value rounded once. */
int oracle_coo_spmv_f32(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row, const int64_t *col,
                        const float *val, float alpha, const float *x, float beta, const float *y0,
                        double *y_out, double *scale_out) {
    int rc = check_range(nrows, ncols, nnz, row, col);
    if (rc) return rc;
    long double *acc = (long double *)calloc((size_t)(nrows > 0 ? nrows : 1), sizeof(long double));
    long double *mag = (long double *)calloc((size_t)(nrows > 0 ? nrows : 1), sizeof(long double));
    if (!acc || !mag) { free(acc); free(mag); return ORACLE_ERR_ALLOC; }
    for (int64_t e = 0; e < nnz; ++e) {
        long double p = (long double)val[e] * (long double)x[col[e]];
        acc[row[e]] += p;
        mag[row[e]] += fabsl(p);
    }
    for (int64_t r = 0; r < nrows; ++r) {
        long double yr = (long double)alpha * acc[r];
        long double sr = fabsl((long double)alpha) * mag[r];
        if (beta != 0.0f) {
            yr += (long double)beta * (long double)y0[r];
            sr += fabsl((long double)beta) * fabsl((long double)y0[r]);
        }
        y_out[r] = (double)yr;
        if (scale_out) scale_out[r] = (double)sr;
    }
    free(acc);
    free(mag);
    return ORACLE_OK;
}

/* Sampled rows: the same definition evaluated only for the rows listed in
 * rows_sel (COO must be sorted by row; row_ptr[r]..row_ptr[r+1] delimit row r).
 * Used for full-size parity on outputs the oracle computes one by one. */
int oracle_rows_spmv_f64(int64_t nsel, const int64_t *rows_sel, const int64_t *row_ptr, const int64_t *col,
                         const double *val, double alpha, const double *x, double beta, const double *y0,
                         double *y_out, double *scale_out) {
    for (int64_t t = 0; t < nsel; ++t) {
        int64_t r = rows_sel[t];
        long double acc = 0.0L, mag = 0.0L;
        for (int64_t e = row_ptr[r]; e < row_ptr[r + 1]; ++e) {
            long double p = (long double)val[e] * (long double)x[col[e]];
            acc += p;
            mag += fabsl(p);
        }
        long double yr = (long double)alpha * acc;
        long double sr = fabsl((long double)alpha) * mag;
        if (beta != 0.0) {
            yr += (long double)beta * (long double)y0[r];
            sr += fabsl((long double)beta) * fabsl((long double)y0[r]);
        }
        y_out[t] = (double)yr;
        if (scale_out) scale_out[t] = (double)sr;
    }
    return ORACLE_OK;
}
