/*
 * Seeded synthetic matrices in C (OpenMP): the same COO, bit for bit, as the
 * numpy generators in gen/matrices.py (stencil, band), which remain the
 * definition -- tests/test_gen.py checks the two against each other. This is
 * input generation only: no CRSD arithmetic lives here. It exists because the
 * BASELINE configurations reach 3.17e9 entries (C5), which numpy generates
 * in minutes on one core.
 *
 * Output order is the numpy order: rows ascending, within a row the stencil
 * displacements by ascending linear offset (= ascending column) / the band
 * offsets ascending.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

static inline uint64_t splitmix64(uint64_t z) {
    z = z + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* gen.matrices.counter_uniform: U[0,1) with 53 bits from (counter, seed) */
static inline double counter_uniform(uint64_t c, uint64_t seed) {
    const uint64_t z = splitmix64((c * 0x2545F4914F6CDD1Dull) ^ seed);
    return (double)(z >> 11) * (1.0 / 9007199254740992.0);
}

typedef struct {
    int64_t n1, n2, n3;
    int32_t m;           /* displacements */
    int32_t di[27], dj[27], dk[27];
    int64_t lin[27];     /* ascending */
    int32_t cq;          /* index of (0,0,0) */
    int32_t present;     /* center = number of present couplings */
    int32_t random;      /* values *= 1 + 0.1 (2u - 1) */
    uint64_t seed;
    int32_t drop;        /* C3 idle blocks (gen.matrices.c3_drop) */
    int64_t k1a, k1b, j2a, j2b, k2a, k2b, k3a, k3b;
} Stencil;

/* entries of row idx into (col, val); returns the count */
static int stencil_row(const Stencil *S, int64_t idx, int64_t *col, double *val) {
    const int64_t i = idx % S->n1, j = (idx / S->n1) % S->n2, k = idx / (S->n1 * S->n2);
    int valid[27];
    int nvalid = 0;
    for (int q = 0; q < S->m; ++q) {
        const int64_t a = i + S->di[q], b = j + S->dj[q], c = k + S->dk[q];
        int v = a >= 0 && a < S->n1 && b >= 0 && b < S->n2 && c >= 0 && c < S->n3;
        if (q != S->cq && S->drop) {
            int d = 0;
            if (S->dk[q] == 1) d |= (k >= S->k1a && k < S->k1b);
            if (S->dj[q] != 0) d |= (j >= S->j2a && j < S->j2b && k >= S->k2a && k < S->k2b);
            d |= (k >= S->k3a && k < S->k3b);
            v &= !d;
        }
        valid[q] = v;
        nvalid += v;
    }
    int n = 0;
    for (int q = 0; q < S->m; ++q) {
        double x = -1.0;
        if (q == S->cq) x = S->present ? (double)(nvalid - 1) : (double)(S->m - 1);
        if (S->random) {
            const double u = counter_uniform((uint64_t)(idx * (int64_t)S->m + q), S->seed);
            double t = 2.0 * u;
            t = t - 1.0;
            t = 0.1 * t;
            t = 1.0 + t;
            x = x * t;
        }
        int v = valid[q];
        if (q == S->cq && S->present) v &= (x != 0.0);
        if (v) {
            if (col) {
                col[n] = idx + S->lin[q];
                val[n] = x;
            }
            ++n;
        }
    }
    return n;
}

/* disp: m x 3 int32 (di, dj, dk), in ascending linear-offset order. drop8:
 * k1a k1b j2a j2b k2a k2b k3a k3b or NULL. Two calls: with col == NULL it
 * returns the entry count; then fills col/val (int64, double) and the COO
 * rows (row, int64[count]) and/or the CSR pointers (ptr, int64[rows + 1],
 * from 0), whichever is not NULL. */
int64_t fg_stencil(int64_t n1, int64_t n2, int64_t n3, int32_t m, const int32_t *disp, int32_t present,
                   int32_t random, uint64_t seed, const int64_t *drop8, int64_t row_begin, int64_t row_end,
                   int64_t *row, int64_t *ptr, int64_t *col, double *val, int32_t nthreads) {
    Stencil S;
    memset(&S, 0, sizeof(S));
    S.n1 = n1;
    S.n2 = n2;
    S.n3 = n3;
    S.m = m;
    S.cq = -1;
    for (int q = 0; q < m; ++q) {
        S.di[q] = disp[3 * q];
        S.dj[q] = disp[3 * q + 1];
        S.dk[q] = disp[3 * q + 2];
        S.lin[q] = S.di[q] + n1 * (S.dj[q] + n2 * S.dk[q]);
        if (!S.di[q] && !S.dj[q] && !S.dk[q]) S.cq = q;
    }
    S.present = present;
    S.random = random;
    S.seed = seed;
    if (drop8) {
        S.drop = 1;
        S.k1a = drop8[0], S.k1b = drop8[1], S.j2a = drop8[2], S.j2b = drop8[3];
        S.k2a = drop8[4], S.k2b = drop8[5], S.k3a = drop8[6], S.k3b = drop8[7];
    }
    const int64_t nr = row_end - row_begin;
    if (nr <= 0) return 0;
    if (nthreads < 1) nthreads = omp_get_max_threads();
    /* blocks of rows: count, prefix, fill */
    const int64_t B = 1 << 16;
    const int64_t nb = (nr + B - 1) / B;
    int64_t *cnt = (int64_t *)calloc((size_t)nb + 1, sizeof(int64_t));
    if (!cnt) return -1;
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
    for (int64_t b = 0; b < nb; ++b) {
        int64_t c = 0;
        const int64_t r1 = row_begin + (b + 1 < nb ? (b + 1) * B : nr);
        for (int64_t r = row_begin + b * B; r < r1; ++r) c += stencil_row(&S, r, NULL, NULL);
        cnt[b + 1] = c;
    }
    for (int64_t b = 0; b < nb; ++b) cnt[b + 1] += cnt[b];
    const int64_t total = cnt[nb];
    if (col) {
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
        for (int64_t b = 0; b < nb; ++b) {
            int64_t e = cnt[b];
            const int64_t r1 = row_begin + (b + 1 < nb ? (b + 1) * B : nr);
            for (int64_t r = row_begin + b * B; r < r1; ++r) {
                const int n = stencil_row(&S, r, col + e, val + e);
                if (row)
                    for (int t = 0; t < n; ++t) row[e + t] = r;
                if (ptr) ptr[r - row_begin] = e;
                e += n;
            }
        }
        if (ptr) ptr[nr] = total;
    }
    free(cnt);
    return total;
}

/* gen.matrices.band: rows [a_k, b_k) carry offsets offs[optr[k]..optr[k+1])
 * (ascending); entries with columns outside [0, n) omitted; value 2u - 1
 * from counter row * 2^20 + (offset + 2^19), 0 replaced by 0.5. */
int64_t fg_band(int64_t n, int32_t nranges, const int64_t *ra, const int64_t *rb, const int64_t *optr,
                const int64_t *offs, uint64_t seed, int64_t row_begin, int64_t row_end, int64_t *row, int64_t *ptr,
                int64_t *col, double *val, int32_t nthreads) {
    if (nthreads < 1) nthreads = omp_get_max_threads();
    int64_t total = 0;
    for (int32_t g = 0; g < nranges; ++g) {
        const int64_t a = ra[g] > row_begin ? ra[g] : row_begin, b = rb[g] < row_end ? rb[g] : row_end;
        if (a >= b) continue;
        const int64_t *o = offs + optr[g];
        const int64_t no = optr[g + 1] - optr[g];
        const int64_t nr = b - a;
        const int64_t B = 1 << 16;
        const int64_t nb = (nr + B - 1) / B;
        int64_t *cnt = (int64_t *)calloc((size_t)nb + 1, sizeof(int64_t));
        if (!cnt) return -1;
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
        for (int64_t k = 0; k < nb; ++k) {
            int64_t c = 0;
            const int64_t r1 = a + (k + 1 < nb ? (k + 1) * B : nr);
            for (int64_t r = a + k * B; r < r1; ++r)
                for (int64_t q = 0; q < no; ++q) c += (r + o[q] >= 0 && r + o[q] < n);
            cnt[k + 1] = c;
        }
        for (int64_t k = 0; k < nb; ++k) cnt[k + 1] += cnt[k];
        if (col) {
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
            for (int64_t k = 0; k < nb; ++k) {
                int64_t e = total + cnt[k];
                const int64_t r1 = a + (k + 1 < nb ? (k + 1) * B : nr);
                for (int64_t r = a + k * B; r < r1; ++r) {
                    if (ptr) ptr[r - row_begin] = e;
                    for (int64_t q = 0; q < no; ++q) {
                        const int64_t c = r + o[q];
                        if (c < 0 || c >= n) continue;
                        double v = 2.0 * counter_uniform((uint64_t)(r * (int64_t)(1 << 20) + (o[q] + (1 << 19))), seed) - 1.0;
                        if (v == 0.0) v = 0.5;
                        if (row) row[e] = r;
                        col[e] = c;
                        val[e] = v;
                        ++e;
                    }
                }
            }
        }
        total += cnt[nb];
        free(cnt);
    }
    /* rows of [row_begin, row_end) outside every range carry no entries */
    if (col && ptr && row_end > row_begin) {
        /* such a row starts where the next row in a range starts */
        int64_t next = total;
        for (int64_t r = row_end - row_begin - 1; r >= 0; --r) {
            int in = 0;
            for (int32_t g = 0; g < nranges; ++g) in |= (row_begin + r >= ra[g] && row_begin + r < rb[g]);
            if (in) next = ptr[r]; else ptr[r] = next;
        }
        ptr[row_end - row_begin] = total;
    }
    return total;
}
