/*
 * Plain-C consumer of the C-ABI (include/crsd.h): no Python, no torch.
 *
 * Builds the 7-point Dirichlet Laplacian (center 6, couplings -1) on an
 * n x n x n grid as COO, creates the CRSD handle, runs y = A x on the GPU and
 * checks it against the closed forms of the oracle:
 * A * 1 has 0 in interior rows and the number of boundary neighbours missing
 * elsewhere; then solves A x = A * ones with crsd_cg and checks x ~ 1.
 *
 * Build (done by __graft_entry__.build()):
 *   gcc -O2 -I include examples/crsd_example.c -L<pkg> -lcrsd -lcudart -o examples/crsd_example
 * Run: examples/crsd_example [n]   (exit code 0 = pass)
 */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <cuda_runtime.h>

#include "crsd.h"

#define CHECK(call)                                                                  \
    do {                                                                             \
        crsd_status_t st_ = (call);                                                  \
        if (st_ != CRSD_OK) {                                                        \
            fprintf(stderr, "%s failed: %d %s\n", #call, (int)st_, crsd_last_error()); \
            return 2;                                                                \
        }                                                                            \
    } while (0)

int main(int argc, char **argv) {
    const int64_t n = argc > 1 ? atoll(argv[1]) : 48;
    const int64_t N = n * n * n;
    int64_t *row = malloc(sizeof(int64_t) * 7 * N), *col = malloc(sizeof(int64_t) * 7 * N);
    double *val = malloc(sizeof(double) * 7 * N);
    int64_t nnz = 0;
    for (int64_t k = 0; k < n; ++k)
        for (int64_t j = 0; j < n; ++j)
            for (int64_t i = 0; i < n; ++i) {
                const int64_t r = i + n * (j + n * k);
                const int64_t d[7][3] = {{0, 0, -1}, {0, -1, 0}, {-1, 0, 0}, {0, 0, 0}, {1, 0, 0}, {0, 1, 0}, {0, 0, 1}};
                for (int q = 0; q < 7; ++q) {
                    const int64_t ii = i + d[q][0], jj = j + d[q][1], kk = k + d[q][2];
                    if (ii < 0 || jj < 0 || kk < 0 || ii >= n || jj >= n || kk >= n) continue;
                    row[nnz] = r;
                    col[nnz] = ii + n * (jj + n * kk);
                    val[nnz] = (q == 3) ? 6.0 : -1.0;
                    ++nnz;
                }
            }
    crsd_matrix_t A = NULL;
    CHECK(crsd_create_from_coo(N, N, nnz, row, col, val, CRSD_R64F, NULL, &A));
    crsd_info_t info;
    CHECK(crsd_get_info(A, &info));

    double *x, *y, *b;
    if (cudaMalloc((void **)&x, sizeof(double) * N) || cudaMalloc((void **)&y, sizeof(double) * N) ||
        cudaMalloc((void **)&b, sizeof(double) * N))
        return 3;
    double *h = malloc(sizeof(double) * N);
    for (int64_t r = 0; r < N; ++r) h[r] = 1.0;
    cudaMemcpy(x, h, sizeof(double) * N, cudaMemcpyHostToDevice);
    const double one = 1.0, zero = 0.0;
    CHECK(crsd_spmv(A, &one, x, &zero, y, NULL));
    cudaMemcpy(h, y, sizeof(double) * N, cudaMemcpyDeviceToHost);
    int64_t bad = 0;
    for (int64_t k = 0; k < n; ++k)
        for (int64_t j = 0; j < n; ++j)
            for (int64_t i = 0; i < n; ++i) {
                /* closed form: A*1 = number of missing neighbours (exact integers) */
                const double expect = (i == 0) + (i == n - 1) + (j == 0) + (j == n - 1) + (k == 0) + (k == n - 1);
                bad += h[i + n * (j + n * k)] != expect;
            }
    printf("spmv: %lld rows, %lld nnz, variant %d, closed-form mismatches %lld\n", (long long)N, (long long)nnz,
           info.variant, (long long)bad);

    /* CG: b = A * 1, x0 = 0 -> x ~ 1 */
    cudaMemcpy(b, y, sizeof(double) * N, cudaMemcpyDeviceToDevice);
    cudaMemset(x, 0, sizeof(double) * N);
    crsd_cg_result_t res;
    CHECK(crsd_cg(A, b, x, 2000, 1e-10, 25, NULL, NULL, &res, NULL));
    cudaMemcpy(h, x, sizeof(double) * N, cudaMemcpyDeviceToHost);
    double err = 0.0;
    for (int64_t r = 0; r < N; ++r) err = fmax(err, fabs(h[r] - 1.0));
    printf("cg: %d steps, converged %d, max |x - 1| = %.3e\n", res.iterations, res.converged, err);
    CHECK(crsd_destroy(A));
    cudaFree(x);
    cudaFree(y);
    cudaFree(b);
    free(row);
    free(col);
    free(val);
    free(h);
    return (bad == 0 && res.converged && err < 1e-8) ? 0 : 1;
}
