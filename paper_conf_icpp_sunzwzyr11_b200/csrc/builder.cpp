// Host CRSD builder: COO/CSR -> CRSD (B200 layout).
//
// Follows PAPER.md §II with the readings of DESIGN.md:
//   1. canonicalise to row-sorted CSR; duplicates rejected or summed;
//      explicit zeros kept as scatter entries (R10)
//   2. per row segment a summary of the diagonals it touches:
//      offset d = col - row, count, first/last row
//   3. presence (R1/R2): d is stored in segment s iff s holds >= 2
//      nonzeros of d, or s meets a run of nonzeros of d whose zero gaps are
//      <= idle_max and which holds >= 2 nonzeros
//   4. maximal runs of segments with equal diagonal sets = the paper's
//      diagonal patterns / Table II instances; distinct sets are
//      deduplicated into the pattern table the kernels read
//   5. values segment-major, diagonal-major, row-minor (address
//      formula P:L613-623), zeros filled; everything else goes to the
//      per-segment scatter list (R5)
// OpenMP over segments; O(nnz) apart from per-row column sorts of unsorted
// input. Shares no code with oracle/.
#include <omp.h>

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstring>
#include <map>
#include <new>

#include "crsd_internal.h"

namespace crsd {

namespace {

inline int64_t floordiv(int64_t a, int64_t b) {  // b > 0
    int64_t q = a / b;
    return (a % b != 0 && a < 0) ? q - 1 : q;
}

struct DiagSum {
    int64_t d;
    int32_t cnt;
    int32_t minl;  // first local row within the segment
    int32_t maxl;  // last local row within the segment
};

// Open-addressing hash from offset to DiagSum, reused per thread.
struct DiagTable {
    std::vector<int64_t> key;
    std::vector<DiagSum> val;
    std::vector<int32_t> used;
    int logcap = 0;
    static constexpr int64_t EMPTY = INT64_MIN;

    void reserve_for(int64_t n) {
        int lc = 6;
        while ((int64_t(1) << lc) < 2 * n + 2) ++lc;
        if (lc > logcap) {
            logcap = lc;
            key.assign(size_t(1) << lc, EMPTY);
            val.resize(size_t(1) << lc);
        }
    }
    inline void add(int64_t d, int32_t l) {
        const uint64_t mask = (uint64_t(1) << logcap) - 1;
        uint64_t h = (uint64_t(d) * 0x9E3779B97F4A7C15ull) >> (64 - logcap);
        for (;; h = (h + 1) & mask) {
            if (key[h] == d) {
                DiagSum &s = val[h];
                s.cnt++;
                if (l < s.minl) s.minl = l;
                if (l > s.maxl) s.maxl = l;
                return;
            }
            if (key[h] == EMPTY) {
                key[h] = d;
                val[h] = DiagSum{d, 1, l, l};
                used.push_back((int32_t)h);
                return;
            }
        }
    }
    void drain(std::vector<DiagSum> &out) {
        out.clear();
        out.reserve(used.size());
        for (int32_t h : used) {
            out.push_back(val[h]);
            key[h] = EMPTY;
        }
        used.clear();
        std::sort(out.begin(), out.end(), [](const DiagSum &a, const DiagSum &b) { return a.d < b.d; });
    }
};

const DiagSum *find_diag(const std::vector<DiagSum> &v, int64_t d) {
    auto it = std::lower_bound(v.begin(), v.end(), d, [](const DiagSum &a, int64_t x) { return a.d < x; });
    return (it != v.end() && it->d == d) ? &*it : nullptr;
}

template <typename T>
inline bool is_zero(T v) {
    return v == T(0);
}

// Canonical CSR over local rows.
template <typename T>
struct CSR {
    std::vector<int64_t> ptr;  // n_local + 1, relative to col/val
    const int64_t *col = nullptr;
    const T *val = nullptr;
    std::vector<int64_t> col_own;
    std::vector<T> val_own;
};

template <typename T>
crsd_status_t canonicalise_coo(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row, const int64_t *col,
                               const T *val, const BuildOptions &o, CSR<T> &C, int64_t &min_col, int64_t &max_col) {
    const int64_t rb = o.row_begin, re = o.row_end, n = re - rb;
    // range check, sortedness, column extent
    int64_t bad = -1;
    bool sorted = true;
    int64_t mn = INT64_MAX, mx = INT64_MIN;
#pragma omp parallel for schedule(static) reduction(&& : sorted) reduction(min : mn) reduction(max : mx)
    for (int64_t e = 0; e < nnz; ++e) {
        const int64_t r = row[e], c = col[e];
        if (r < rb || r >= re || c < 0 || c >= ncols) {
#pragma omp atomic write
            bad = e;
        }
        if (c < mn) mn = c;
        if (c > mx) mx = c;
        if (e > 0 && (row[e - 1] > r || (row[e - 1] == r && col[e - 1] >= c))) sorted = false;
    }
    if (bad >= 0) {
        return fail(CRSD_ERR_INDEX_RANGE, "COO entry " + std::to_string(bad) + " (" + std::to_string(row[bad]) + "," +
                                              std::to_string(col[bad]) + ") outside rows [" + std::to_string(rb) +
                                              "," + std::to_string(re) + ") x cols [0," + std::to_string(ncols) + ")");
    }
    min_col = nnz ? mn : 0;
    max_col = nnz ? mx : -1;
    C.ptr.assign(n + 1, 0);
    if (sorted) {
        // strictly sorted by (row, col): no duplicates; CSR pointers by boundaries
        C.col = col;
        C.val = val;
        int64_t *ptr = C.ptr.data();
#pragma omp parallel for schedule(static)
        for (int64_t e = 0; e < nnz; ++e) {
            const int64_t r = row[e] - rb;
            const int64_t rp = (e == 0) ? -1 : row[e - 1] - rb;
            for (int64_t q = rp + 1; q <= r; ++q) ptr[q] = e;
        }
        const int64_t last = nnz ? row[nnz - 1] - rb : -1;
        for (int64_t q = last + 1; q <= n; ++q) ptr[q] = nnz;
        return CRSD_OK;
    }
    // counting sort by row (stable), then per-row stable sort by column
    std::vector<int64_t> cnt(n + 1, 0);
    for (int64_t e = 0; e < nnz; ++e) cnt[row[e] - rb + 1]++;
    for (int64_t q = 0; q < n; ++q) cnt[q + 1] += cnt[q];
    std::vector<int64_t> cur(cnt.begin(), cnt.end() - 1);
    std::vector<int64_t> ctmp(nnz);
    std::vector<T> vtmp(nnz);
    for (int64_t e = 0; e < nnz; ++e) {
        const int64_t p = cur[row[e] - rb]++;
        ctmp[p] = col[e];
        vtmp[p] = val[e];
    }
    cur.clear();
    cur.shrink_to_fit();
    bool dup = false;
    int64_t dup_row = -1, dup_col = -1;
    std::vector<int64_t> ucnt(n + 1, 0);
#pragma omp parallel
    {
        std::vector<std::pair<int64_t, T>> buf;
#pragma omp for schedule(dynamic, 4096)
        for (int64_t q = 0; q < n; ++q) {
            const int64_t b = cnt[q], e = cnt[q + 1];
            bool ok = true;
            for (int64_t i = b + 1; i < e; ++i)
                if (ctmp[i - 1] >= ctmp[i]) { ok = false; break; }
            if (!ok) {
                buf.clear();
                for (int64_t i = b; i < e; ++i) buf.emplace_back(ctmp[i], vtmp[i]);
                std::stable_sort(buf.begin(), buf.end(),
                                 [](const std::pair<int64_t, T> &a, const std::pair<int64_t, T> &c) { return a.first < c.first; });
                for (int64_t i = b; i < e; ++i) {
                    ctmp[i] = buf[i - b].first;
                    vtmp[i] = buf[i - b].second;
                }
            }
            int64_t u = (e > b) ? 1 : 0;
            for (int64_t i = b + 1; i < e; ++i) {
                if (ctmp[i] == ctmp[i - 1]) {
                    if (!(o.flags & CRSD_SUM_DUPLICATES)) {
#pragma omp critical
                        {
                            dup = true;
                            dup_row = q + rb;
                            dup_col = ctmp[i];
                        }
                    }
                } else {
                    ++u;
                }
            }
            ucnt[q + 1] = u;
        }
    }
    if (dup)
        return fail(CRSD_ERR_DUPLICATE, "duplicate COO entry (" + std::to_string(dup_row) + "," + std::to_string(dup_col) +
                                            ") (set CRSD_SUM_DUPLICATES to sum)");
    for (int64_t q = 0; q < n; ++q) ucnt[q + 1] += ucnt[q];
    if (ucnt[n] == nnz) {
        C.col_own.swap(ctmp);
        C.val_own.swap(vtmp);
        C.ptr.swap(cnt);
    } else {  // sum duplicates in input order (stable sort kept it)
        C.col_own.resize(ucnt[n]);
        C.val_own.resize(ucnt[n]);
#pragma omp parallel for schedule(dynamic, 4096)
        for (int64_t q = 0; q < n; ++q) {
            int64_t w = ucnt[q] - 1;
            for (int64_t i = cnt[q]; i < cnt[q + 1]; ++i) {
                if (i > cnt[q] && ctmp[i] == ctmp[i - 1]) {
                    C.val_own[w] += vtmp[i];
                } else {
                    ++w;
                    C.col_own[w] = ctmp[i];
                    C.val_own[w] = vtmp[i];
                }
            }
        }
        C.ptr.swap(ucnt);
    }
    C.col = C.col_own.data();
    C.val = C.val_own.data();
    return CRSD_OK;
}

template <typename T>
crsd_status_t build_from_csr_t(int64_t nrows, int64_t ncols, CSR<T> &C, const BuildOptions &o, HostCRSD &H) {
    const int64_t rb = o.row_begin, n = o.row_end - o.row_begin;
    const int32_t m = o.mrows;
    const int64_t nseg = (n + m - 1) / m;
    const int64_t reach = int64_t(o.idle_max) + 1;  // two nonzeros a<b on d share a piece iff b-a <= reach
    const bool drop_zeros = (o.flags & CRSD_DROP_ZEROS) != 0;
    H.nrows = nrows;
    H.ncols = ncols;
    H.row_begin = rb;
    H.row_end = o.row_end;
    H.n_local = n;
    H.mrows = m;
    H.idle_max = o.idle_max;
    H.elem = sizeof(T);
    H.nseg = nseg;
    const int64_t *ptr = C.ptr.data();
    const int64_t *col = C.col;
    const T *val = C.val;

    // ---- step 2: per-segment diagonal summaries ----
    std::vector<std::vector<DiagSum>> sums(nseg);
#pragma omp parallel
    {
        DiagTable tab;
#pragma omp for schedule(dynamic, 16)
        for (int64_t s = 0; s < nseg; ++s) {
            const int64_t r0 = s * m, r1 = std::min<int64_t>(n, r0 + m);
            tab.reserve_for(ptr[r1] - ptr[r0]);
            for (int64_t r = r0; r < r1; ++r) {
                const int64_t grow = rb + r;
                for (int64_t e = ptr[r]; e < ptr[r + 1]; ++e)
                    if (!is_zero(val[e])) tab.add(col[e] - grow, int32_t(r - r0));
            }
            tab.drain(sums[s]);
        }
    }

    // ---- step 3: presence rule ----
    std::vector<std::vector<int64_t>> pres(nseg);
#pragma omp parallel for schedule(dynamic, 64)
    for (int64_t s = 0; s < nseg; ++s) {
        auto &P = pres[s];
        for (const DiagSum &ds : sums[s]) {
            if (ds.cnt >= 2) {
                P.push_back(ds.d);
                continue;
            }
            // singleton: is its nearest neighbour along d within reach?
            const int64_t r = s * m + ds.minl;
            bool in_piece = false;
            for (int64_t t = s - 1; t >= 0; --t) {
                if (r - (t * m + m - 1) > reach) break;
                if (const DiagSum *q = find_diag(sums[t], ds.d)) {
                    in_piece = (r - (t * m + q->maxl) <= reach);
                    break;
                }
            }
            if (!in_piece) {
                for (int64_t t = s + 1; t < nseg; ++t) {
                    if (t * m - r > reach) break;
                    if (const DiagSum *q = find_diag(sums[t], ds.d)) {
                        in_piece = (t * m + q->minl - r <= reach);
                        break;
                    }
                }
            }
            if (in_piece) P.push_back(ds.d);
        }
    }
    if (o.idle_max >= m) {
        // empty segments inside a bridged run (only possible when idle_max >= mrows)
        std::vector<std::pair<int64_t, int64_t>> extra;
        for (int64_t s = 0; s < nseg; ++s) {
            for (const DiagSum &ds : sums[s]) {
                const int64_t last = s * m + ds.maxl;
                for (int64_t t = s + 1; t < nseg; ++t) {
                    if (t * m - last > reach) break;
                    if (const DiagSum *q = find_diag(sums[t], ds.d)) {
                        if (t >= s + 2 && t * m + q->minl - last <= reach)
                            for (int64_t u = s + 1; u < t; ++u) extra.emplace_back(u, ds.d);
                        break;
                    }
                }
            }
        }
        for (auto &pr : extra) pres[pr.first].push_back(pr.second);
        if (!extra.empty()) {
#pragma omp parallel for schedule(dynamic, 64)
            for (int64_t s = 0; s < nseg; ++s) {
                std::sort(pres[s].begin(), pres[s].end());
                pres[s].erase(std::unique(pres[s].begin(), pres[s].end()), pres[s].end());
            }
        }
    }
    sums.clear();
    sums.shrink_to_fit();

    // ---- step 4: instances and distinct patterns ----
    std::map<std::vector<int64_t>, int32_t> pid;
    H.pat_ptr.assign(1, 0);
    H.pat_offsets.clear();
    H.inst.clear();
    std::vector<int32_t> seg_inst(nseg);
    int64_t slots = 0;
    for (int64_t s = 0; s < nseg; ++s) {
        if (s == 0 || pres[s] != pres[s - 1]) {
            auto it = pid.find(pres[s]);
            int32_t p;
            if (it == pid.end()) {
                p = (int32_t)pid.size();
                pid.emplace(pres[s], p);
                H.pat_offsets.insert(H.pat_offsets.end(), pres[s].begin(), pres[s].end());
                H.pat_ptr.push_back((int64_t)H.pat_offsets.size());
            } else {
                p = it->second;
            }
            H.inst.push_back(Instance{s, 0, p, slots});
        }
        Instance &I = H.inst.back();
        I.nseg++;
        slots += (int64_t)pres[s].size() * m;
        seg_inst[s] = (int32_t)H.inst.size() - 1;
    }
    pres.clear();
    pres.shrink_to_fit();
    H.nslots = slots;

    // ---- step 5: values and scatter list ----
    try {
        H.vals.assign((size_t)slots * sizeof(T), 0);
    } catch (const std::bad_alloc &) {
        return fail(CRSD_ERR_ALLOC, "host allocation of " + std::to_string(slots * (int64_t)sizeof(T)) + " bytes failed");
    }
    T *V = reinterpret_cast<T *>(H.vals.data());
    H.scat_ptr.assign(nseg + 1, 0);
    int64_t ndiag = 0;
    auto seg_base = [&](int64_t s, const int64_t *&offs, int64_t &nd) {
        const Instance &I = H.inst[seg_inst[s]];
        offs = H.pat_offsets.data() + H.pat_ptr[I.pattern];
        nd = H.pat_ptr[I.pattern + 1] - H.pat_ptr[I.pattern];
        return I.val_base + (s - I.first_seg) * nd * m;
    };
    // pass A: store diagonal values, count scatter
#pragma omp parallel for schedule(dynamic, 16) reduction(+ : ndiag)
    for (int64_t s = 0; s < nseg; ++s) {
        const int64_t *offs;
        int64_t nd;
        const int64_t base = seg_base(s, offs, nd);
        const int64_t r0 = s * m, r1 = std::min<int64_t>(n, r0 + m);
        int64_t ns = 0;
        for (int64_t r = r0; r < r1; ++r) {
            const int64_t grow = rb + r;
            int64_t j = 0;
            for (int64_t e = ptr[r]; e < ptr[r + 1]; ++e) {
                const T v = val[e];
                if (is_zero(v) && drop_zeros) continue;
                const int64_t d = col[e] - grow;
                while (j < nd && offs[j] < d) ++j;
                if (j < nd && offs[j] == d && !is_zero(v)) {
                    V[base + j * m + (r - r0)] = v;
                    ++ndiag;
                } else {
                    ++ns;
                }
            }
        }
        H.scat_ptr[s + 1] = ns;
    }
    for (int64_t s = 0; s < nseg; ++s) H.scat_ptr[s + 1] += H.scat_ptr[s];
    const int64_t nscat = H.scat_ptr[nseg];
    H.ndiag_nnz = ndiag;
    H.nnz = ndiag + nscat;
    H.scat_row.resize(nscat);
    H.scat_col.resize(nscat);
    H.scat_val.resize((size_t)nscat * sizeof(T));
    T *SV = reinterpret_cast<T *>(H.scat_val.data());
    // pass B: scatter entries in (row, col) order
#pragma omp parallel for schedule(dynamic, 16)
    for (int64_t s = 0; s < nseg; ++s) {
        if (H.scat_ptr[s + 1] == H.scat_ptr[s]) continue;
        const int64_t *offs;
        int64_t nd;
        seg_base(s, offs, nd);
        const int64_t r0 = s * m, r1 = std::min<int64_t>(n, r0 + m);
        int64_t w = H.scat_ptr[s];
        for (int64_t r = r0; r < r1; ++r) {
            const int64_t grow = rb + r;
            int64_t j = 0;
            for (int64_t e = ptr[r]; e < ptr[r + 1]; ++e) {
                const T v = val[e];
                if (is_zero(v) && drop_zeros) continue;
                const int64_t d = col[e] - grow;
                while (j < nd && offs[j] < d) ++j;
                if (!(j < nd && offs[j] == d && !is_zero(v))) {
                    H.scat_row[w] = int32_t(r - r0);
                    H.scat_col[w] = col[e];
                    SV[w] = v;
                    ++w;
                }
            }
        }
    }
    // pass C (CRSD_PAPER_ELL): the paper's scatter storage --
    // every row with a scatter point, whole (all its entries, ascending
    // columns), in ELL: column-major, width = the longest such row, padding
    // col -1 / value 0 (Bell & Garland ELL; R6)
    H.paper_ell = (o.flags & CRSD_PAPER_ELL) != 0;
    if (H.paper_ell) {
        std::vector<int64_t> rows;
        for (int64_t s = 0; s < nseg; ++s)
            for (int64_t e = H.scat_ptr[s]; e < H.scat_ptr[s + 1]; ++e) {
                const int64_t r = s * m + H.scat_row[e];
                if (rows.empty() || rows.back() != r) rows.push_back(r);
            }
        auto row_len = [&](int64_t r) {
            int64_t k = 0;
            for (int64_t e = ptr[r]; e < ptr[r + 1]; ++e) k += !(drop_zeros && is_zero(val[e]));
            return k;
        };
        int64_t W = 0;
        for (int64_t r : rows) W = std::max(W, row_len(r));
        const int64_t N = (int64_t)rows.size();
        H.ell_nrows = N;
        H.ell_width = W;
        H.ell_rowno = rows;
        H.ell_col.assign((size_t)(N * W), -1);
        H.ell_val.assign((size_t)(N * W) * sizeof(T), 0);
        T *EV = reinterpret_cast<T *>(H.ell_val.data());
        for (int64_t i = 0; i < N; ++i) {
            const int64_t r = rows[i];
            int64_t k = 0;
            for (int64_t e = ptr[r]; e < ptr[r + 1]; ++e) {
                if (drop_zeros && is_zero(val[e])) continue;
                H.ell_col[k * N + i] = col[e];
                EV[k * N + i] = val[e];
                ++k;
            }
        }
    }
    return CRSD_OK;
}

crsd_status_t check_common(int64_t nrows, int64_t ncols, const BuildOptions &o) {
    if (nrows <= 0 || ncols <= 0) return fail(CRSD_ERR_INVALID_ARG, "nrows and ncols must be > 0");
    if (nrows >= (int64_t(1) << 31) || ncols >= (int64_t(1) << 31))
        return fail(CRSD_ERR_UNSUPPORTED, "nrows and ncols must be < 2^31 (32-bit diagonal offsets)");
    if (o.mrows < 1 || o.mrows > 65536) return fail(CRSD_ERR_INVALID_ARG, "mrows must be in [1, 65536]");
    if (o.row_begin < 0 || o.row_end > nrows || o.row_begin >= o.row_end)
        return fail(CRSD_ERR_INVALID_ARG, "row range [row_begin,row_end) invalid");
    if (o.row_begin % o.mrows != 0) return fail(CRSD_ERR_INVALID_ARG, "row_begin must be a multiple of mrows");
    return CRSD_OK;
}

}  // namespace

crsd_status_t build_from_coo(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row, const int64_t *col,
                             const void *val, crsd_dtype_t dtype, const BuildOptions &o, HostCRSD &H) {
    crsd_status_t st = check_common(nrows, ncols, o);
    if (st) return st;
    if (nnz < 0) return fail(CRSD_ERR_INVALID_ARG, "nnz must be >= 0");
    if (nnz > 0 && (!row || !col || !val)) return fail(CRSD_ERR_INVALID_ARG, "row/col/val must not be NULL");
    if (o.nthreads > 0) omp_set_num_threads(o.nthreads);
    H.dtype = dtype;
    try {
        if (dtype == CRSD_R64F) {
            CSR<double> C;
            st = canonicalise_coo<double>(nrows, ncols, nnz, row, col, (const double *)val, o, C, H.min_col_ref,
                                          H.max_col_ref);
            if (st) return st;
            return build_from_csr_t<double>(nrows, ncols, C, o, H);
        } else if (dtype == CRSD_R32F) {
            CSR<float> C;
            st = canonicalise_coo<float>(nrows, ncols, nnz, row, col, (const float *)val, o, C, H.min_col_ref,
                                         H.max_col_ref);
            if (st) return st;
            return build_from_csr_t<float>(nrows, ncols, C, o, H);
        }
    } catch (const std::bad_alloc &) {
        return fail(CRSD_ERR_ALLOC, "host allocation failed in the CRSD builder");
    }
    return fail(CRSD_ERR_INVALID_ARG, "dtype must be CRSD_R32F or CRSD_R64F");
}

crsd_status_t build_from_csr(int64_t nrows, int64_t ncols, const int64_t *row_ptr, const int64_t *col,
                             const void *val, crsd_dtype_t dtype, const BuildOptions &o, HostCRSD &H) {
    crsd_status_t st = check_common(nrows, ncols, o);
    if (st) return st;
    if (!row_ptr) return fail(CRSD_ERR_INVALID_ARG, "row_ptr must not be NULL");
    const int64_t n = o.row_end - o.row_begin;
    const int64_t b = row_ptr[0], nnz = row_ptr[n] - b;
    if (nnz < 0) return fail(CRSD_ERR_INVALID_ARG, "row_ptr not nondecreasing");
    for (int64_t q = 0; q < n; ++q)
        if (row_ptr[q + 1] < row_ptr[q]) return fail(CRSD_ERR_INVALID_ARG, "row_ptr not nondecreasing");
    if (o.nthreads > 0) omp_set_num_threads(o.nthreads);
    // Canonical input (columns strictly increasing in every row, all in
    // range): the builder reads the caller's arrays in place -- no copy of
    // the entries (C5 at full size is 3.17e9 of them).
    {
        bool canon = true;
        int64_t mn = INT64_MAX, mx = INT64_MIN;
#pragma omp parallel for schedule(dynamic, 4096) reduction(&& : canon) reduction(min : mn) reduction(max : mx)
        for (int64_t q = 0; q < n; ++q)
            for (int64_t e = row_ptr[q]; e < row_ptr[q + 1]; ++e) {
                const int64_t c = col[e];
                if (c < 0 || c >= ncols || (e > row_ptr[q] && col[e - 1] >= c)) canon = false;
                if (c < mn) mn = c;
                if (c > mx) mx = c;
            }
        if (canon) {
            H.dtype = dtype;
            H.min_col_ref = nnz ? mn : 0;
            H.max_col_ref = nnz ? mx : -1;
            try {
                if (dtype == CRSD_R64F) {
                    CSR<double> C;
                    C.ptr.resize(n + 1);
                    for (int64_t q = 0; q <= n; ++q) C.ptr[q] = row_ptr[q] - b;
                    C.col = col + b;
                    C.val = (const double *)val + b;
                    return build_from_csr_t<double>(nrows, ncols, C, o, H);
                } else if (dtype == CRSD_R32F) {
                    CSR<float> C;
                    C.ptr.resize(n + 1);
                    for (int64_t q = 0; q <= n; ++q) C.ptr[q] = row_ptr[q] - b;
                    C.col = col + b;
                    C.val = (const float *)val + b;
                    return build_from_csr_t<float>(nrows, ncols, C, o, H);
                }
                return fail(CRSD_ERR_INVALID_ARG, "dtype must be CRSD_R32F or CRSD_R64F");
            } catch (const std::bad_alloc &) {
                return fail(CRSD_ERR_ALLOC, "host allocation failed in the CRSD builder");
            }
        }
    }
    // otherwise expand to COO rows and reuse the COO path (one canonicalisation:
    // range errors, column sort, duplicates)
    std::vector<int64_t> rows;
    try {
        rows.resize(nnz);
    } catch (const std::bad_alloc &) {
        return fail(CRSD_ERR_ALLOC, "host allocation failed");
    }
#pragma omp parallel for schedule(static)
    for (int64_t q = 0; q < n; ++q)
        for (int64_t e = row_ptr[q]; e < row_ptr[q + 1]; ++e) rows[e - b] = o.row_begin + q;
    const size_t es = dtype == CRSD_R64F ? 8 : 4;
    return build_from_coo(nrows, ncols, nnz, rows.data(), col + b, (const char *)val + es * b, dtype, o, H);
}

// ---------------------------------------------------------------------------
// kernel-facing layout helpers
// ---------------------------------------------------------------------------
static void seg_pattern(const HostCRSD &H, int64_t s, const Instance *&I) {
    // instances are sorted by first_seg
    auto it = std::upper_bound(H.inst.begin(), H.inst.end(), s,
                               [](int64_t v, const Instance &a) { return v < a.first_seg; });
    I = &*(it - 1);
}

void segment_x_window(const HostCRSD &H, int64_t s, int rpt, int64_t &lo, int64_t &hi) {
    const Instance *I;
    seg_pattern(H, s, I);
    const int64_t nd = H.ndias(I->pattern);
    const int64_t row0 = s * H.mrows;
    if (nd == 0) {
        lo = row0;
        hi = row0;
        return;
    }
    const int64_t omin = H.pat_offsets[H.pat_ptr[I->pattern]];
    const int64_t omax = H.pat_offsets[H.pat_ptr[I->pattern + 1] - 1];
    lo = row0 + rpt * floordiv(omin, rpt);
    hi = row0 + H.mrows + rpt * (floordiv(omax, rpt) + 1);
}

void needed_halo(const HostCRSD &H, int rpt, int64_t &need_lo, int64_t &need_hi) {
    int64_t lo = 0, hi = H.n_local;
    for (int64_t s = 0; s < H.nseg; ++s) {
        int64_t a, b;
        segment_x_window(H, s, rpt, a, b);
        if (a < b) {
            lo = std::min(lo, a);
            hi = std::max(hi, b);
        }
    }
    for (int64_t c : H.scat_col) {
        lo = std::min(lo, c - H.row_begin);
        hi = std::max(hi, c - H.row_begin + 1);
    }
    need_lo = -lo;
    need_hi = hi - H.n_local;
}

void make_segdescs(const HostCRSD &H, int rpt, int64_t x_lo, int64_t x_hi, std::vector<SegDesc> &out) {
    out.resize(H.nseg);
    const int64_t m = H.mrows;
    for (size_t i = 0; i < H.inst.size(); ++i) {
        const Instance &I = H.inst[i];
        const int64_t nd = H.ndias(I.pattern);
        for (int64_t s = I.first_seg; s < I.first_seg + I.nseg; ++s) {
            SegDesc &D = out[s];
            D.val_base = I.val_base + (s - I.first_seg) * nd * m;
            D.scat_begin = H.scat_ptr[s];
            D.nscat = (int32_t)(H.scat_ptr[s + 1] - H.scat_ptr[s]);
            D.off_begin = (int32_t)H.pat_ptr[I.pattern];
            D.ndias = (uint16_t)nd;
            D.plan_begin = 0;
            int64_t lo, hi;
            segment_x_window(H, s, rpt, lo, hi);
            int32_t f = 0;
            const bool partial = (s * m + m > H.n_local);
            if (partial || (lo < hi && (lo < x_lo || hi > x_hi))) f |= SEG_EDGE;
            // boundary: reads x outside the owned range [0, n_local) (after
            // clipping to the valid range, which is what guarded loads read)
            const int64_t clo = std::max(lo, x_lo), chi = std::min(hi, x_hi);
            bool bnd = (clo < chi) && (clo < 0 || chi > H.n_local);
            for (int64_t e = H.scat_ptr[s]; e < H.scat_ptr[s + 1] && !bnd; ++e) {
                const int64_t c = H.scat_col[e] - H.row_begin;
                if (c < 0 || c >= H.n_local) bnd = true;
            }
            if (bnd) f |= SEG_BOUNDARY;
            D.flags = (uint16_t)f;
        }
    }
}

int64_t make_plans(const HostCRSD &H, int64_t gap, std::vector<int32_t> &plan, std::vector<SegDesc> &segs,
                   int64_t *xmax_elems) {
    int64_t xmx = 0;
    const int64_t m = H.mrows, es = H.elem, al = 16 / H.elem;  // alignment in elements
    std::vector<int32_t> begin(H.npat());
    std::vector<int64_t> smem(H.npat());
    plan.clear();
    int64_t mx = 0;
    for (int64_t p = 0; p < H.npat(); ++p) {
        const int64_t *o = H.pat_offsets.data() + H.pat_ptr[p];
        const int64_t nd = H.pat_ptr[p + 1] - H.pat_ptr[p];
        // clusters of offsets closer than `gap`: one x window each
        std::vector<std::pair<int64_t, int64_t>> win;  // (start, count) in elements, aligned
        std::vector<int32_t> xoff(nd), xwin(nd);
        int64_t xbase = 0;
        for (int64_t d = 0; d < nd;) {
            int64_t e = d;
            while (e + 1 < nd && o[e + 1] - o[e] <= gap) ++e;
            const int64_t st = floordiv(o[d], al) * al;
            const int64_t en = (floordiv(m - 1 + o[e], al) + 1) * al;
            for (int64_t q = d; q <= e; ++q) {
                xoff[q] = (int32_t)(xbase + o[q] - st);
                xwin[q] = (int32_t)win.size();
            }
            win.emplace_back(st, en - st);
            xbase += en - st;
            d = e + 1;
        }
        begin[p] = (int32_t)plan.size();
        xmx = std::max(xmx, xbase);
        const int64_t bytes = nd * m * es + xbase * es;
        smem[p] = bytes;
        mx = std::max(mx, bytes);
        plan.push_back((int32_t)win.size());
        plan.push_back((int32_t)std::min<int64_t>(bytes, INT32_MAX));
        for (auto &w : win) {
            plan.push_back((int32_t)w.first);
            plan.push_back((int32_t)w.second);
        }
        plan.insert(plan.end(), xoff.begin(), xoff.end());
        plan.insert(plan.end(), xwin.begin(), xwin.end());
    }
    if (plan.empty()) plan.push_back(0);
    if (xmax_elems) *xmax_elems = xmx;
    for (size_t i = 0; i < H.inst.size(); ++i) {
        const Instance &I = H.inst[i];
        for (int64_t s = I.first_seg; s < I.first_seg + I.nseg; ++s) segs[s].plan_begin = begin[I.pattern];
    }
    return mx;
}

}  // namespace crsd
