// C-ABI of libcrsd (include/crsd.h): handle lifetime, device upload,
// single-GPU SpMV, host end-to-end SpMV, introspection.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "crsd_internal.h"
#include "crsd_handle.h"

namespace crsd {

static thread_local std::string g_err;

void set_error(const std::string &msg) { g_err = msg; }

crsd_status_t fail(crsd_status_t st, const std::string &msg) {
    g_err = msg;
    return st;
}

crsd_status_t cuda_fail(cudaError_t e, const char *what) {
    return fail(CRSD_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

#define CUDA_TRY(expr)                                       \
    do {                                                     \
        cudaError_t _e = (expr);                             \
        if (_e != cudaSuccess) return cuda_fail(_e, #expr); \
    } while (0)

static crsd_status_t dev_alloc_copy(void **dptr, const void *src, size_t bytes, int64_t &counter) {
    *dptr = nullptr;
    if (bytes == 0) return CRSD_OK;
    cudaError_t e = cudaMalloc(dptr, bytes);
    if (e != cudaSuccess) {
        *dptr = nullptr;
        return fail(e == cudaErrorMemoryAllocation ? CRSD_ERR_ALLOC : CRSD_ERR_CUDA,
                    "cudaMalloc(" + std::to_string(bytes) + "): " + cudaGetErrorString(e));
    }
    counter += (int64_t)bytes;
    if (src) CUDA_TRY(cudaMemcpy(*dptr, src, bytes, cudaMemcpyHostToDevice));
    return CRSD_OK;
}

void free_device(crsd_matrix_s *A) {
    jit_free(A);
    if (A->e2e_ready) {
        if (A->device >= 0) cudaSetDevice(A->device);
        cudaStreamSynchronize((cudaStream_t)A->e2e_h2d);
        cudaStreamSynchronize((cudaStream_t)A->e2e_d2h);
        for (void *e : A->e2e_ev_x) cudaEventDestroy((cudaEvent_t)e);
        for (void *e : A->e2e_ev_y) cudaEventDestroy((cudaEvent_t)e);
        cudaEventDestroy((cudaEvent_t)A->e2e_ev_start);
        cudaEventDestroy((cudaEvent_t)A->e2e_ev_done);
        cudaStreamDestroy((cudaStream_t)A->e2e_h2d);
        cudaStreamDestroy((cudaStream_t)A->e2e_d2h);
        A->e2e_ready = false;
    }
    if (A->device >= 0) cudaSetDevice(A->device);
    if (A->cg_stream) {
        cudaStreamSynchronize((cudaStream_t)A->cg_stream);
        cudaStreamDestroy((cudaStream_t)A->cg_stream);
        cudaEventDestroy((cudaEvent_t)A->cg_ev_in);
        cudaEventDestroy((cudaEvent_t)A->cg_ev_out);
        A->cg_stream = A->cg_ev_in = A->cg_ev_out = nullptr;
    }
    // direct-mode padded x (crsd_dist_x_alloc): unmap the peers', free mine
    for (crsd_matrix_s::DirectX &d : A->dx) {
        for (void *p : d.peer)
            if (p) cudaIpcCloseMemHandle(p);
        if (d.own) cudaFree(d.own);
    }
    A->dx.clear();
    void *ptrs[] = {A->d_vals, A->d_segs, A->d_offs, A->d_plan, A->d_scat_row, A->d_scat_col, A->d_scat_val, A->d_scat_rec,
                    A->d_scat_slab, A->d_list_interior, A->d_list_boundary, A->d_list_all_edge, A->d_x_scratch, A->d_y_scratch, A->d_cg,
                    A->d_ell_rowno, A->d_ell_col, A->d_ell_val};
    for (void *p : ptrs)
        if (p) cudaFree(p);
    A->d_vals = A->d_segs = A->d_offs = A->d_plan = A->d_scat_row = A->d_scat_col = A->d_scat_val = A->d_scat_rec = A->d_scat_slab = nullptr;
    A->d_list_interior = A->d_list_boundary = A->d_list_all_edge = A->d_x_scratch = A->d_y_scratch = A->d_cg = nullptr;
    A->d_ell_rowno = A->d_ell_col = A->d_ell_val = nullptr;
    A->cg_bytes = 0;
}

// Layout of x for this handle: valid range and halo widths (DESIGN.md
// "Multi-GPU"), segment descriptors and work lists.
static void plan_layout(crsd_matrix_s *A) {
    HostCRSD &H = A->H;
    if (!H.partitioned) {
        A->halo_lo = A->halo_hi = A->halo_lo_valid = A->halo_hi_valid = 0;
        A->x_lo = 0;
        A->x_hi = H.ncols;
    } else {
        int64_t need_lo, need_hi;
        needed_halo(H, A->rpt, need_lo, need_hi);
        A->halo_lo_valid = std::min<int64_t>(H.row_begin, std::max<int64_t>(0, need_lo));
        A->halo_hi_valid = std::min<int64_t>(H.ncols - H.row_end, std::max<int64_t>(0, need_hi));
        A->halo_lo = (A->halo_lo_valid + 3) / 4 * 4;
        A->halo_hi = (A->halo_hi_valid + 3) / 4 * 4;
        A->x_lo = -A->halo_lo_valid;
        A->x_hi = H.n_local + A->halo_hi_valid;
    }
    make_segdescs(H, A->rpt, A->x_lo, A->x_hi, A->segdesc);
    // x windows: offsets closer than mrows share one staged window (merging
    // two windows whose gap is below mrows never adds bytes, and every window
    // is one bulk copy: fewer, larger copies)
    A->smem_bytes = make_plans(H, H.mrows, A->plan, A->segdesc, &A->xmax_elems);
    // TMA variant shape: smallest split of a segment into row slices whose
    // staging (values + x windows) stays <= 40 KB, i.e. >= 5 CTAs per SM
    A->tma_split = 1;
    A->tma_smem = A->smem_bytes;
    for (int split = 1; split <= 8; split *= 2) {
        const int64_t rc = H.mrows / split;
        if (H.mrows % split || rc % 32 || (rc * H.elem) % 16) break;
        int64_t mx = 0;
        for (const Instance &I : H.inst) {
            const int64_t p = I.pattern;
            // plan of pattern p: [nwin, bytes, (st, cnt) x nwin, ...]
            const int32_t *pl = A->plan.data() + A->segdesc[I.first_seg].plan_begin;
            int64_t el = H.ndias((int32_t)p) * rc;
            for (int w = 0; w < pl[0]; ++w) el += pl[3 + 2 * w] - (H.mrows - rc);
            mx = std::max(mx, el * H.elem);
        }
        A->tma_split = split;
        A->tma_smem = mx;
        if (mx <= 40 * 1024) break;
    }
    {
        // rows per thread: the vector width of the dtype (2 fp64, 4 fp32) as
        // long as a CTA keeps >= 2 warps
        const int64_t rc = H.mrows / A->tma_split;
        int q = A->rpt;
        while (q > 1 && rc / q < 64) q /= 2;
        while (rc / q > 256) q *= 2;  // <= 256 threads per CTA
        A->tma_q = q;
    }
    A->list_interior.clear();
    A->list_boundary.clear();
    A->nedge = 0;
    for (int64_t s = 0; s < H.nseg; ++s) {
        const SegDesc &D = A->segdesc[s];
        if (D.flags & SEG_EDGE) A->nedge++;
        if (D.flags & SEG_BOUNDARY) A->list_boundary.push_back((int32_t)s);
        else A->list_interior.push_back((int32_t)s);
    }
}

bool slab_ok(const crsd_matrix_s *A) {
    const HostCRSD &H = A->H;
    if (H.nscatter() == 0 || (A->tune & CRSD_TUNE_JIT_NO_SLAB) || H.mrows > 65535) return false;
    for (int64_t c : H.scat_col)
        if (c - H.row_begin < INT32_MIN || c - H.row_begin > INT32_MAX) return false;
    return true;
}

static crsd_status_t upload(crsd_matrix_s *A) {
    HostCRSD &H = A->H;
    if (A->device < 0) CUDA_TRY(cudaGetDevice(&A->device));
    CUDA_TRY(cudaSetDevice(A->device));
    CUDA_TRY(cudaDeviceGetAttribute(&A->sm_count, cudaDevAttrMultiProcessorCount, A->device));
    int64_t &cnt = A->device_bytes;
    crsd_status_t st;
    if ((st = dev_alloc_copy(&A->d_vals, H.vals.data(), H.vals.size(), cnt))) return st;
    if ((st = dev_alloc_copy(&A->d_segs, A->segdesc.data(), A->segdesc.size() * sizeof(SegDesc), cnt))) return st;
    std::vector<int32_t> offs32(H.pat_offsets.begin(), H.pat_offsets.end());
    if (offs32.empty()) offs32.push_back(0);
    if ((st = dev_alloc_copy(&A->d_offs, offs32.data(), offs32.size() * 4, cnt))) return st;
    if ((st = dev_alloc_copy(&A->d_plan, A->plan.data(), A->plan.size() * 4, cnt))) return st;
    const int64_t ns = H.nscatter();
    std::vector<int64_t> colrel(ns);
    for (int64_t e = 0; e < ns; ++e) colrel[e] = H.scat_col[e] - H.row_begin;
    if ((st = dev_alloc_copy(&A->d_scat_row, H.scat_row.data(), ns * 4, cnt))) return st;
    if ((st = dev_alloc_copy(&A->d_scat_col, colrel.data(), ns * 8, cnt))) return st;
    if ((st = dev_alloc_copy(&A->d_scat_val, H.scat_val.data(), H.scat_val.size(), cnt))) return st;
    {
        std::vector<ScatRec> rec(ns);
        for (int64_t e = 0; e < ns; ++e) {
            ScatRec r{};
            r.col = colrel[e];
            r.row = H.scat_row[e];
            std::memcpy(&r.val, H.scat_val.data() + e * H.elem, H.elem);
            rec[e] = r;
        }
        if ((st = dev_alloc_copy(&A->d_scat_rec, rec.data(), ns * sizeof(ScatRec), cnt))) return st;
    }
    // scatter slab (JIT codelets; CRSD_TUNE_JIT_NO_SLAB keeps the descriptor path)
    if (slab_ok(A)) {
        std::vector<SlabRec> sl((size_t)H.nseg * SLAB_K);
        for (int64_t sg = 0; sg < H.nseg; ++sg) {
            const int64_t b = H.scat_ptr[sg], n = H.scat_ptr[sg + 1] - b;
            for (int l = 0; l < SLAB_K; ++l) {
                SlabRec r{};
                r.n = (uint16_t)std::min<int64_t>(n, 65535);
                if (l < n) {
                    r.col = (int32_t)colrel[b + l];
                    r.row = (uint16_t)H.scat_row[b + l];
                    std::memcpy(&r.val, H.scat_val.data() + (b + l) * H.elem, H.elem);
                }
                sl[sg * SLAB_K + l] = r;
            }
        }
        if ((st = dev_alloc_copy(&A->d_scat_slab, sl.data(), sl.size() * sizeof(SlabRec), cnt))) return st;
    }
    if ((st = dev_alloc_copy(&A->d_list_interior, A->list_interior.data(), A->list_interior.size() * 4, cnt))) return st;
    if ((st = dev_alloc_copy(&A->d_list_boundary, A->list_boundary.data(), A->list_boundary.size() * 4, cnt))) return st;
    if (H.paper_ell && H.ell_nrows > 0) {
        if ((st = dev_alloc_copy(&A->d_ell_rowno, H.ell_rowno.data(), H.ell_rowno.size() * 8, cnt))) return st;
        if ((st = dev_alloc_copy(&A->d_ell_col, H.ell_col.data(), H.ell_col.size() * 8, cnt))) return st;
        if ((st = dev_alloc_copy(&A->d_ell_val, H.ell_val.data(), H.ell_val.size(), cnt))) return st;
    }
    // the host copy of the bulk arrays is dropped after upload (export reads the device copy)
    std::vector<uint8_t>().swap(H.vals);
    std::vector<uint8_t>().swap(H.scat_val);
    A->host_vals_dropped = true;
    return CRSD_OK;
}

static int auto_variant(const crsd_matrix_s *A, bool jit, bool pipe_fits) {
    if (jit && A->smem_bytes <= 75 * 1024) return VARIANT_JIT;
    if (A->tma_split == 1 && A->tma_smem <= 32 * 1024) return VARIANT_TMA;
    if (pipe_fits && A->H.mrows <= 1024) return VARIANT_PIPE;
    return VARIANT_LDG;
}

static crsd_status_t finish_create(crsd_matrix_s *A, const crsd_opts_t &o, crsd_matrix_t *out) {
    A->rpt = (A->H.dtype == CRSD_R64F) ? 2 : 4;
    int64_t maxnd = 0;
    for (int64_t p = 0; p < A->H.npat(); ++p) maxnd = std::max<int64_t>(maxnd, A->H.ndias((int32_t)p));
    if (maxnd > MAX_NDIAS) {
        delete A;
        return fail(CRSD_ERR_UNSUPPORTED, "a pattern has more than " + std::to_string(MAX_NDIAS) + " diagonals");
    }
    plan_layout(A);
    const int64_t smem_cap = 200 * 1024;
    if (o.variant == CRSD_VARIANT_TMA && A->tma_smem > smem_cap) {
        const std::string msg = "TMA variant: staging needs " + std::to_string(A->tma_smem) +
                                " bytes of shared memory per CTA (> 200 KB); use CRSD_VARIANT_LDG";
        delete A;
        return fail(CRSD_ERR_UNSUPPORTED, msg);
    }
    // PIPE needs two x slots of the largest pattern's windows plus >= 2 ring stages
    const int64_t pipe_need = 2 * A->xmax_elems * A->H.elem + 2 * 8 * (int64_t)A->H.mrows * A->H.elem + 1024;
    if (o.variant == CRSD_VARIANT_PIPE && pipe_need > smem_cap) {
        const std::string msg = "PIPE variant: x staging needs " + std::to_string(pipe_need) +
                                " bytes of shared memory per CTA (> 200 KB); use CRSD_VARIANT_LDG";
        delete A;
        return fail(CRSD_ERR_UNSUPPORTED, msg);
    }
    if (o.variant == CRSD_VARIANT_PIPE && A->H.mrows > 1024) {
        delete A;
        return fail(CRSD_ERR_UNSUPPORTED, "PIPE variant: mrows must be <= 1024");
    }
    A->jit_chunk = o.jit_chunk;
    A->tune = o.tune;
    A->e2e_chunks = o.e2e_chunks;  // 0: chosen from the vector size at the first crsd_spmv_host
    const bool auto_jit = !(o.tune & CRSD_TUNE_NO_JIT);
    if (o.variant == CRSD_VARIANT_JIT) A->variant = VARIANT_JIT;
    else if (o.variant == CRSD_VARIANT_LDG) A->variant = VARIANT_LDG;
    else if (o.variant == CRSD_VARIANT_TMA) A->variant = VARIANT_TMA;
    else if (o.variant == CRSD_VARIANT_PIPE) A->variant = VARIANT_PIPE;
    else {
        // AUTO, from the variant sweeps in profiles/r01_sweep*.jsonl. The
        // runtime-generated one-shot kernel (JIT: every pattern quantity a
        // literal, a whole segment staged per CTA, scatter points gathered
        // while the bulk copies fly) leads wherever a segment stages in <= 75
        // KB (>= 3 CTAs per SM): C2 1.05 / 1.02, C3 0.95 / 0.99 of the
        // measured copy peak (fp64 / fp32, sweep18), ahead of the table-driven
        // TMA (C2 0.98 / 0.90) and of the persistent ring (PIPE, C3 0.90 /
        // 0.85), which remains the choice for bigger segments; the register
        // variant when neither staging fits in shared memory. Without NVRTC
        // the JIT falls back to TMA (small segments) below.
        A->variant = auto_variant(A, auto_jit, pipe_need <= smem_cap);
    }
    if (!A->host_only) {
        if (A->H.mrows / A->rpt > 256) {
            delete A;
            return fail(CRSD_ERR_UNSUPPORTED, "GPU path needs mrows / RPT <= 256 threads per CTA (mrows <= 512 fp64, 1024 fp32)");
        }
        if (A->H.mrows % (32 * A->rpt) != 0) {
            delete A;
            return fail(CRSD_ERR_UNSUPPORTED, "GPU path needs mrows % (32*RPT) == 0 (RPT = 2 fp64, 4 fp32); got mrows=" +
                                                  std::to_string(o.mrows) + " (use CRSD_HOST_ONLY for inspection)");
        }
        crsd_status_t st = upload(A);
        if (!st && A->variant == VARIANT_JIT) {
            st = jit_build(A);
            if (st == CRSD_ERR_UNSUPPORTED && o.variant == CRSD_VARIANT_AUTO) {
                A->variant = auto_variant(A, false, pipe_need <= smem_cap);  // no NVRTC
                st = CRSD_OK;
            }
        }
        if (st) {
            free_device(A);
            delete A;
            return st;
        }
    }
    *out = A;
    return CRSD_OK;
}

static crsd_status_t resolve_opts(int64_t nrows, crsd_dtype_t dtype, const crsd_opts_t *opts, crsd_opts_t &o,
                                  BuildOptions &b) {
    if (opts) o = *opts;
    else crsd_opts_init(&o);
    // default: 2 KB per diagonal run of a segment (256 fp64, 512 fp32)
    if (o.mrows == 0) o.mrows = (dtype == CRSD_R64F) ? 256 : 512;
    if (o.idle_max < 0) o.idle_max = o.mrows - 1;
    if (o.row_begin == 0 && o.row_end == 0) o.row_end = nrows;
    b.mrows = o.mrows;
    b.idle_max = o.idle_max;
    b.flags = o.flags;
    b.row_begin = o.row_begin;
    b.row_end = o.row_end;
    b.nthreads = o.nthreads;
    return CRSD_OK;
}

template <typename T>
static crsd_status_t run_spmv(crsd_matrix_s *A, T alpha, const T *x, T beta, T *y, const int32_t *list,
                              int64_t seg_begin, int64_t count, void *stream, int &launches, const HaloSync *halo,
                              bool pdl) {
    if (count <= 0) return CRSD_OK;
    SpmvArgs<T> a;
    a.halo = halo;
    a.pdl = pdl;
    a.vals = (const T *)A->d_vals;
    a.segs = (const SegDesc *)A->d_segs;
    a.pat_offs = (const int32_t *)A->d_offs;
    a.plan = (const int32_t *)A->d_plan;
    a.smem_bytes = (int32_t)A->smem_bytes;
    a.tma_split = A->tma_split;
    a.tma_q = A->tma_q;
    a.tma_smem = A->tma_smem;
    a.has_scatter = A->H.nscatter() > 0;
    a.pipe_xmax_elems = (int32_t)A->xmax_elems;
    {
        int64_t mx = 0;
        for (int64_t p = 0; p < A->H.npat(); ++p) mx = std::max<int64_t>(mx, A->H.ndias((int32_t)p));
        a.max_ndias = (int32_t)mx;
    }
    a.variant = A->variant;
    a.scat_row = (const int32_t *)A->d_scat_row;
    a.scat_col = (const int64_t *)A->d_scat_col;
    a.scat_val = (const T *)A->d_scat_val;
    a.scat_rec = (const ScatRec *)A->d_scat_rec;
    a.scat_slab = (const SlabRec *)A->d_scat_slab;
    a.x = x;
    a.x_lo = A->x_lo;
    a.x_hi = A->x_hi;
    a.y = y;
    a.nrows = A->H.n_local;
    a.seg_list = list;
    a.seg_begin = seg_begin;
    a.seg_count = count;
    a.mrows = A->H.mrows;
    a.alpha = alpha;
    a.beta = beta;
    int n = A->variant == VARIANT_JIT ? jit_launch<T>(A, a, stream) : launch_spmv<T>(a, A->sm_count, stream);
    if (n <= -10000)
        return fail(CRSD_ERR_CUDA, std::string("cudaFuncSetAttribute(MaxDynamicSharedMemorySize=") +
                                       std::to_string(a.smem_bytes) + "): " + cudaGetErrorString((cudaError_t)(-n - 10000)));
    if (n < 0)
        return fail(CRSD_ERR_CUDA, std::string("kernel launch (variant ") + std::to_string(a.variant) + ", grid " +
                                       std::to_string(a.seg_count) + ", block " + std::to_string(A->H.mrows / A->rpt) +
                                       ", smem " + std::to_string(a.variant == VARIANT_TMA ? a.tma_smem : 0) +
                                       "): " + cudaGetErrorString((cudaError_t)(-n)));
    launches += n;
    return CRSD_OK;
}

crsd_status_t run_lists(crsd_matrix_s *A, const void *alpha, const void *x_base, const void *beta, void *y,
                        const int32_t *list, int64_t seg_begin, int64_t count, void *stream, int &launches,
                        const HaloSync *halo, bool pdl) {
    if (halo && A->variant != VARIANT_JIT) return fail(CRSD_ERR_UNSUPPORTED, "fused halo receive needs the JIT variant");
    if (A->H.dtype == CRSD_R64F)
        return run_spmv<double>(A, *(const double *)alpha, (const double *)x_base, *(const double *)beta, (double *)y,
                                list, seg_begin, count, stream, launches, halo, pdl);
    return run_spmv<float>(A, *(const float *)alpha, (const float *)x_base, *(const float *)beta, (float *)y, list,
                           seg_begin, count, stream, launches, halo, pdl);
}

}  // namespace crsd

using namespace crsd;

extern "C" {

const char *crsd_last_error(void) { return g_err.c_str(); }

const char *crsd_version(void) { return "crsd-b200 0.1 (sm_100a)"; }

crsd_status_t crsd_opts_init(crsd_opts_t *o) {
    if (!o) return fail(CRSD_ERR_INVALID_ARG, "opts is NULL");
    std::memset(o, 0, sizeof(*o));
    o->mrows = 0;
    o->idle_max = -1;
    o->device = -1;
    return CRSD_OK;
}

static crsd_status_t create_common(int64_t nrows, int64_t ncols, crsd_dtype_t dtype, const crsd_opts_t *opts,
                                   crsd_matrix_t *out, bool csr, int64_t nnz, const int64_t *row_or_ptr,
                                   const int64_t *col, const void *val) {
    NvtxRange nv("crsd_create");
    if (!out) return fail(CRSD_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (dtype != CRSD_R32F && dtype != CRSD_R64F) return fail(CRSD_ERR_INVALID_ARG, "bad dtype");
    crsd_opts_t o;
    BuildOptions b;
    resolve_opts(nrows, dtype, opts, o, b);
    crsd_matrix_s *A = new (std::nothrow) crsd_matrix_s();
    if (!A) return fail(CRSD_ERR_ALLOC, "handle allocation failed");
    A->host_only = (o.flags & CRSD_HOST_ONLY) != 0;
    A->device = o.device;
    A->H.partitioned = !(o.row_begin == 0 && o.row_end == nrows);
    crsd_status_t st = csr ? build_from_csr(nrows, ncols, row_or_ptr, col, val, dtype, b, A->H)
                           : build_from_coo(nrows, ncols, nnz, row_or_ptr, col, val, dtype, b, A->H);
    // AUTO height for fp32: 512 rows (2 KB per diagonal run) unless a
    // segment's staging (values + x windows) would then leave fewer than 4
    // CTAs per SM -- then 256. Measured (profiles/r02/sweep1*): C3 f32
    // (27 diagonals, 70 KB at 512 -> 3 CTAs/SM) 1.06 of the copy peak at
    // 256 against 1.02 at 512; C4 f32 (19 diagonals, 56 KB -> 4 CTAs/SM) and
    // C2 f32 keep 512 (round 1 sweep19: 256 costs them 0.17-0.3).
    const bool auto_m = (!opts || opts->mrows == 0) && dtype == CRSD_R32F && (o.row_begin % 256) == 0;
    if (!st && auto_m && A->H.mrows == 512) {
        std::vector<int32_t> pl;
        std::vector<SegDesc> sg(A->H.nseg);
        const int64_t mx = make_plans(A->H, A->H.mrows, pl, sg);
        const int64_t per_cta = (mx + 127) / 128 * 128 + 1024 + 256;
        if ((228 * 1024) / per_cta < 4) {
            A->H = HostCRSD();
            o.mrows = b.mrows = 256;
            if (!opts || opts->idle_max < 0) o.idle_max = b.idle_max = 255;
            st = csr ? build_from_csr(nrows, ncols, row_or_ptr, col, val, dtype, b, A->H)
                     : build_from_coo(nrows, ncols, nnz, row_or_ptr, col, val, dtype, b, A->H);
        }
    }
    if (st) {
        delete A;
        return st;
    }
    A->H.partitioned = !(o.row_begin == 0 && o.row_end == nrows);
    if (A->H.partitioned && (o.flags & CRSD_PAPER_ELL)) {
        delete A;
        return fail(CRSD_ERR_UNSUPPORTED, "CRSD_PAPER_ELL needs a one-GPU (non-partitioned) handle");
    }
    if (A->H.partitioned && nrows != ncols) {
        delete A;
        return fail(CRSD_ERR_UNSUPPORTED, "row-partitioned handles need a square matrix");
    }
    return finish_create(A, o, out);
}

crsd_status_t crsd_create_from_coo(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row, const int64_t *col,
                                   const void *val, crsd_dtype_t dtype, const crsd_opts_t *opts, crsd_matrix_t *out) {
    return create_common(nrows, ncols, dtype, opts, out, false, nnz, row, col, val);
}

crsd_status_t crsd_create_from_csr(int64_t nrows, int64_t ncols, const int64_t *row_ptr, const int64_t *col,
                                   const void *val, crsd_dtype_t dtype, const crsd_opts_t *opts, crsd_matrix_t *out) {
    return create_common(nrows, ncols, dtype, opts, out, true, 0, row_ptr, col, val);
}

crsd_status_t crsd_destroy(crsd_matrix_t A) {
    if (!A) return CRSD_OK;
    free_device(A);
    delete A;
    return CRSD_OK;
}

static crsd_status_t check_vec(const void *p, const char *name) {
    if (!p) return fail(CRSD_ERR_INVALID_ARG, std::string(name) + " is NULL");
    if (((uintptr_t)p) & 15) return fail(CRSD_ERR_INVALID_ARG, std::string(name) + " must be 16-byte aligned");
    return CRSD_OK;
}

crsd_status_t crsd_spmv(crsd_matrix_t A, const void *alpha, const void *x, const void *beta, void *y, void *stream) {
    NvtxRange nv("crsd_spmv");
    if (!A) return fail(CRSD_ERR_INVALID_ARG, "A is NULL");
    if (A->host_only) return fail(CRSD_ERR_UNSUPPORTED, "host-only handle");
    if (A->H.partitioned) return fail(CRSD_ERR_UNSUPPORTED, "row-partitioned handle: use crsd_spmv_dist");
    if (!alpha || !beta) return fail(CRSD_ERR_INVALID_ARG, "alpha/beta NULL");
    crsd_status_t st;
    if ((st = check_vec(x, "x")) || (st = check_vec(y, "y"))) return st;
    if (x == y) return fail(CRSD_ERR_INVALID_ARG, "x and y must not alias");
    const bool beta_nz = (A->H.dtype == CRSD_R64F) ? (*(const double *)beta != 0.0) : (*(const float *)beta != 0.0f);
    if (A->H.paper_ell && beta_nz)
        return fail(CRSD_ERR_UNSUPPORTED, "CRSD_PAPER_ELL handles compute y = alpha*A*x (beta must be 0): the ELL part overwrites y");
    int launches = 0;
    cudaSetDevice(A->device);
    const int64_t nseg = A->H.nseg;
    st = run_lists(A, alpha, x, beta, y, nullptr, 0, nseg, stream, launches, nullptr, true);
    if (!st && A->H.paper_ell && A->H.ell_nrows > 0) {
        // second part of the paper's kernel: the scatter rows,
        // stored whole in ELL, overwrite what the diagonal part wrote
        const int e = A->H.dtype == CRSD_R64F
                          ? launch_paper_ell<double>((const int64_t *)A->d_ell_rowno, (const int64_t *)A->d_ell_col,
                                                     (const double *)A->d_ell_val, A->H.ell_nrows, A->H.ell_width,
                                                     (const double *)x, (double *)y, *(const double *)alpha, stream)
                          : launch_paper_ell<float>((const int64_t *)A->d_ell_rowno, (const int64_t *)A->d_ell_col,
                                                    (const float *)A->d_ell_val, A->H.ell_nrows, A->H.ell_width,
                                                    (const float *)x, (float *)y, *(const float *)alpha, stream);
        if (e) st = fail(CRSD_ERR_CUDA, std::string("paper ELL kernel launch: ") + cudaGetErrorString((cudaError_t)e));
        else ++launches;
    }
    A->last_launches = launches;
    return st;
}

// End-to-end SpMV with host vectors, pipelined: x is copied in row-aligned
// chunks on an H2D stream, each row chunk of segments runs as soon as the x
// chunks its windows reach have landed, and its y chunk is copied back on a
// D2H stream while later chunks compute (PCIe is full duplex). This answers
// the paper's transfer caveat by overlapping transfers with
// the SpMV instead of serialising copy -> kernel -> copy.
static crsd_status_t e2e_setup(crsd_matrix_s *A) {
    HostCRSD &H = A->H;
    const int64_t nseg = H.nseg;
    // pipeline depth: fill (the first x chunks) and drain (the last y chunk)
    // cost ~2 chunks of transfer, every chunk ~17 us of per-copy overhead
    // (profiles/r01_e2e_chunk_probe*: C2's 134 MB x is best at 12-16
    // chunks); large vectors get chunks of ~56 MB, at most 64 (C5: 3.6 GB)
    int64_t want = A->e2e_chunks;
    if (want <= 0) want = std::min<int64_t>(64, std::max<int64_t>(16, (H.ncols * H.elem) / (56 << 20)));
    int nch = (int)std::min<int64_t>(want, std::max<int64_t>(1, nseg / 32));
    A->e2e_nchunk = nch;
    A->e2e_seg.resize(nch + 1);
    A->e2e_xcut.resize(nch + 1);
    for (int c = 0; c <= nch; ++c) A->e2e_seg[c] = nseg * c / nch;
    // highest x element each row chunk reads (vector windows, clipped to
    // [0, ncols) as the guarded edge path does, and scatter columns)
    std::vector<int64_t> hi(nch, 0);
    for (int c = 0; c < nch; ++c) {
        for (int64_t sg = A->e2e_seg[c]; sg < A->e2e_seg[c + 1]; ++sg) {
            int64_t lo_w, hi_w;
            segment_x_window(H, sg, A->rpt, lo_w, hi_w);
            if (lo_w < hi_w) hi[c] = std::max(hi[c], std::min(hi_w, H.ncols));
            for (int64_t e = H.scat_ptr[sg]; e < H.scat_ptr[sg + 1]; ++e) hi[c] = std::max(hi[c], H.scat_col[e] + 1);
        }
    }
    // x chunks are aligned with the row chunks, so row chunk c usually waits
    // for x chunk c+1 (its far diagonals reach a few rows into it). Cutting x
    // where each row chunk's reads end instead lets y copies start one chunk
    // earlier but measured slower: the earlier D2H overlaps more of the H2D
    // stream and slows it (C2 f64, 12-16 chunks: 3.38 vs 3.56-3.59 ms;
    // profiles/r01_e2e_cut_ab.txt).
    A->e2e_xcut[0] = 0;
    for (int c = 0; c < nch; ++c) {
        const int64_t xc = std::min<int64_t>(H.ncols, A->e2e_seg[c + 1] * H.mrows) / 4 * 4;
        A->e2e_xcut[c + 1] = std::max(A->e2e_xcut[c], xc);
    }
    A->e2e_xcut[nch] = H.ncols;
    A->e2e_need.assign(nch, 0);
    for (int c = 0; c < nch; ++c) {
        int j = 0;
        while (j < nch - 1 && A->e2e_xcut[j + 1] < hi[c]) ++j;
        A->e2e_need[c] = j;
    }
    cudaStream_t h, d;
    CUDA_TRY(cudaStreamCreateWithFlags(&h, cudaStreamNonBlocking));
    CUDA_TRY(cudaStreamCreateWithFlags(&d, cudaStreamNonBlocking));
    A->e2e_h2d = h;
    A->e2e_d2h = d;
    A->e2e_ev_x.resize(nch);
    A->e2e_ev_y.resize(nch);
    for (int c = 0; c < nch; ++c) {
        cudaEvent_t e1, e2;
        CUDA_TRY(cudaEventCreateWithFlags(&e1, cudaEventDisableTiming));
        CUDA_TRY(cudaEventCreateWithFlags(&e2, cudaEventDisableTiming));
        A->e2e_ev_x[c] = e1;
        A->e2e_ev_y[c] = e2;
    }
    cudaEvent_t e0, e3;
    CUDA_TRY(cudaEventCreateWithFlags(&e0, cudaEventDisableTiming));
    CUDA_TRY(cudaEventCreateWithFlags(&e3, cudaEventDisableTiming));
    A->e2e_ev_start = e0;
    A->e2e_ev_done = e3;
    A->e2e_ready = true;
    return CRSD_OK;
}

crsd_status_t crsd_spmv_host(crsd_matrix_t A, const void *alpha, const void *x_host, const void *beta, void *y_host,
                             void *stream) {
    NvtxRange nv("crsd_spmv_host");
    if (!A) return fail(CRSD_ERR_INVALID_ARG, "A is NULL");
    if (A->host_only) return fail(CRSD_ERR_UNSUPPORTED, "host-only handle");
    if (A->H.partitioned) return fail(CRSD_ERR_UNSUPPORTED, "row-partitioned handle");
    if (A->H.paper_ell) return fail(CRSD_ERR_UNSUPPORTED, "CRSD_PAPER_ELL handle: use crsd_spmv");
    if (!x_host || !y_host || !alpha || !beta) return fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    CUDA_TRY(cudaSetDevice(A->device));
    const size_t es = A->H.elem;
    const size_t xb = A->H.ncols * es, yb = A->H.nrows * es;
    int64_t dummy = 0;
    crsd_status_t st;
    if (!A->d_x_scratch) {
        if ((st = dev_alloc_copy(&A->d_x_scratch, nullptr, xb, dummy))) return st;
        if ((st = dev_alloc_copy(&A->d_y_scratch, nullptr, yb, dummy))) return st;
        A->device_bytes += dummy;
    }
    if (!A->e2e_ready && (st = e2e_setup(A))) return st;
    cudaStream_t s = (cudaStream_t)stream, h = (cudaStream_t)A->e2e_h2d, d = (cudaStream_t)A->e2e_d2h;
    const bool beta_nz = (A->H.dtype == CRSD_R64F) ? (*(const double *)beta != 0.0) : (*(const float *)beta != 0.0f);
    const int nch = A->e2e_nchunk;
    const int64_t m = A->H.mrows;
    char *dx = (char *)A->d_x_scratch, *dy = (char *)A->d_y_scratch;
    const char *hx = (const char *)x_host;
    char *hy = (char *)y_host;
    auto yrange = [&](int c, int64_t &r0, int64_t &r1) {
        r0 = A->e2e_seg[c] * m;
        r1 = std::min<int64_t>(A->H.nrows, A->e2e_seg[c + 1] * m);
    };
    CUDA_TRY(cudaEventRecord((cudaEvent_t)A->e2e_ev_start, s));
    CUDA_TRY(cudaStreamWaitEvent(h, (cudaEvent_t)A->e2e_ev_start, 0));
    CUDA_TRY(cudaStreamWaitEvent(d, (cudaEvent_t)A->e2e_ev_start, 0));
    for (int c = 0; c < nch; ++c) {
        const int64_t x0 = A->e2e_xcut[c], x1 = A->e2e_xcut[c + 1];
        if (x1 > x0) CUDA_TRY(cudaMemcpyAsync(dx + x0 * es, hx + x0 * es, (x1 - x0) * es, cudaMemcpyHostToDevice, h));
        if (beta_nz) {
            int64_t r0, r1;
            yrange(c, r0, r1);
            if (r1 > r0) CUDA_TRY(cudaMemcpyAsync(dy + r0 * es, hy + r0 * es, (r1 - r0) * es, cudaMemcpyHostToDevice, h));
        }
        CUDA_TRY(cudaEventRecord((cudaEvent_t)A->e2e_ev_x[c], h));
    }
    int launches = 0;
    for (int c = 0; c < nch; ++c) {
        const int need = std::max(A->e2e_need[c], beta_nz ? c : 0);
        CUDA_TRY(cudaStreamWaitEvent(s, (cudaEvent_t)A->e2e_ev_x[need], 0));
        st = run_lists(A, alpha, dx, beta, dy, nullptr, A->e2e_seg[c], A->e2e_seg[c + 1] - A->e2e_seg[c], s, launches);
        if (st) return st;
        CUDA_TRY(cudaEventRecord((cudaEvent_t)A->e2e_ev_y[c], s));
        CUDA_TRY(cudaStreamWaitEvent(d, (cudaEvent_t)A->e2e_ev_y[c], 0));
        int64_t r0, r1;
        yrange(c, r0, r1);
        if (r1 > r0) CUDA_TRY(cudaMemcpyAsync(hy + r0 * es, dy + r0 * es, (r1 - r0) * es, cudaMemcpyDeviceToHost, d));
    }
    // all x chunks must have landed before the scratch can be reused (the
    // last row chunk may not need the last x chunk)
    CUDA_TRY(cudaStreamWaitEvent(d, (cudaEvent_t)A->e2e_ev_x[nch - 1], 0));
    CUDA_TRY(cudaEventRecord((cudaEvent_t)A->e2e_ev_done, d));
    CUDA_TRY(cudaStreamWaitEvent(s, (cudaEvent_t)A->e2e_ev_done, 0));
    A->last_launches = launches;
    CUDA_TRY(cudaStreamSynchronize(s));
    return CRSD_OK;
}

crsd_status_t crsd_get_info(crsd_matrix_t A, crsd_info_t *I) {
    if (!A || !I) return fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    const HostCRSD &H = A->H;
    std::memset(I, 0, sizeof(*I));
    I->nrows = H.nrows;
    I->ncols = H.ncols;
    I->row_begin = H.row_begin;
    I->row_end = H.row_end;
    I->mrows = H.mrows;
    I->idle_max = H.idle_max;
    I->dtype = H.dtype;
    I->rows_per_thread = A->rpt;
    I->nnz = H.nnz;
    I->nseg = H.nseg;
    I->ninst = (int64_t)H.inst.size();
    I->npat = H.npat();
    I->noffsets = (int64_t)H.pat_offsets.size();
    int64_t mx = 0;
    for (int64_t p = 0; p < H.npat(); ++p) mx = std::max<int64_t>(mx, H.ndias((int32_t)p));
    I->max_ndias = mx;
    I->nslots = H.nslots;
    I->ndiag_nnz = H.ndiag_nnz;
    I->nfills = H.nslots - H.ndiag_nnz;
    I->nscatter = H.nscatter();
    I->nedge_seg = A->nedge;
    I->halo_lo = A->halo_lo;
    I->halo_hi = A->halo_hi;
    I->halo_lo_valid = A->halo_lo_valid;
    I->halo_hi_valid = A->halo_hi_valid;
    I->device_bytes = A->device_bytes;
    I->variant = A->variant;
    I->smem_bytes = (int32_t)(A->variant == VARIANT_TMA ? A->tma_smem : A->smem_bytes);
    // algorithmic bytes: stored slots + scatter
    // (value + row + col) + x once + y written (+ y read when beta != 0)
    const int64_t es = H.elem;
    const int64_t xs = H.partitioned ? H.n_local : H.ncols;
    const int64_t base = H.nslots * es + I->nscatter * (es + 4 + 8) + xs * es + H.n_local * es;
    I->unique_bytes_beta0 = base;
    I->unique_bytes_beta1 = base + H.n_local * es;
    I->jit_launches = A->variant == VARIANT_JIT ? (int32_t)std::max<size_t>(1, A->jit_ranges.size()) : 1;
    I->pdl = (A->variant == VARIANT_JIT && !A->host_only && jit_pdl(A)) ? 1 : 0;
    I->regstage = (A->variant == VARIANT_JIT && A->jit_rs_function) ? 1 : 0;
    return CRSD_OK;
}

crsd_status_t crsd_export(crsd_matrix_t A, crsd_export_t *E) {
    if (!A || !E) return fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    const HostCRSD &H = A->H;
    for (size_t i = 0; i < H.inst.size(); ++i) {
        if (E->inst_first_seg) E->inst_first_seg[i] = H.inst[i].first_seg;
        if (E->inst_nseg) E->inst_nseg[i] = H.inst[i].nseg;
        if (E->inst_pattern) E->inst_pattern[i] = H.inst[i].pattern;
    }
    if (E->pat_ptr) std::copy(H.pat_ptr.begin(), H.pat_ptr.end(), E->pat_ptr);
    if (E->pat_offsets) std::copy(H.pat_offsets.begin(), H.pat_offsets.end(), E->pat_offsets);
    if (E->scat_ptr) std::copy(H.scat_ptr.begin(), H.scat_ptr.end(), E->scat_ptr);
    if (E->scat_row) std::copy(H.scat_row.begin(), H.scat_row.end(), E->scat_row);
    if (E->scat_col) std::copy(H.scat_col.begin(), H.scat_col.end(), E->scat_col);
    const size_t vb = (size_t)H.nslots * H.elem, sb = (size_t)H.nscatter() * H.elem;
    if (A->host_vals_dropped) {
        cudaSetDevice(A->device);
        if (E->vals && vb) CUDA_TRY(cudaMemcpy(E->vals, A->d_vals, vb, cudaMemcpyDeviceToHost));
        if (E->scat_val && sb) CUDA_TRY(cudaMemcpy(E->scat_val, A->d_scat_val, sb, cudaMemcpyDeviceToHost));
    } else {
        if (E->vals && vb) std::memcpy(E->vals, H.vals.data(), vb);
        if (E->scat_val && sb) std::memcpy(E->scat_val, H.scat_val.data(), sb);
    }
    return CRSD_OK;
}

// Runtime autotuning of the kernel variant (the
// paper leaves such choices to "the property of matrices"):
// every variant whose staging fits is timed on the caller's vectors and the
// fastest becomes the handle's variant.
crsd_status_t crsd_autotune(crsd_matrix_t A, const void *x, void *y, int32_t reps, double *ms_out, int32_t *chosen,
                            void *stream) {
    if (!A) return fail(CRSD_ERR_INVALID_ARG, "A is NULL");
    if (A->host_only) return fail(CRSD_ERR_UNSUPPORTED, "host-only handle");
    if (A->H.partitioned) return fail(CRSD_ERR_UNSUPPORTED, "row-partitioned handle");
    crsd_status_t st;
    if ((st = check_vec(x, "x")) || (st = check_vec(y, "y"))) return st;
    if (x == y) return fail(CRSD_ERR_INVALID_ARG, "x and y must not alias");
    if (reps <= 0) reps = 20;
    // (CRSD_PAPER_ELL: only the diagonal-part kernel is tuned; the ELL pass is fixed)
    CUDA_TRY(cudaSetDevice(A->device));
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t smem_cap = 200 * 1024;
    const int64_t pipe_need = 2 * A->xmax_elems * A->H.elem + 2 * 8 * (int64_t)A->H.mrows * A->H.elem + 1024;
    const int original = A->variant;
    double best = 1e300;
    int best_v = original;
    cudaEvent_t e0, e1;
    CUDA_TRY(cudaEventCreate(&e0));
    CUDA_TRY(cudaEventCreate(&e1));
    const double one_d = 1.0, zero_d = 0.0;
    const float one_f = 1.0f, zero_f = 0.0f;
    const bool f64 = A->H.dtype == CRSD_R64F;
    const void *one = f64 ? (const void *)&one_d : (const void *)&one_f;
    const void *zero = f64 ? (const void *)&zero_d : (const void *)&zero_f;
    for (int v = VARIANT_LDG; v <= VARIANT_JIT; ++v) {
        double ms = -1.0;
        bool ok = true;
        if (v == VARIANT_TMA) ok = A->tma_smem <= smem_cap;
        if (v == VARIANT_PIPE) ok = pipe_need <= smem_cap && A->H.mrows <= 1024;
        if (v == VARIANT_JIT) {
            ok = A->smem_bytes <= smem_cap;
            if (ok && !A->jit_function) ok = jit_build(A) == CRSD_OK;
        }
        if (ok) {
            A->variant = v;
            int l = 0;
            st = CRSD_OK;
            for (int i = 0; i < 3 && !st; ++i) st = run_lists(A, one, x, zero, y, nullptr, 0, A->H.nseg, s, l);
            if (!st) CUDA_TRY(cudaEventRecord(e0, s));
            for (int i = 0; i < reps && !st; ++i) st = run_lists(A, one, x, zero, y, nullptr, 0, A->H.nseg, s, l);
            if (!st) {
                CUDA_TRY(cudaEventRecord(e1, s));
                CUDA_TRY(cudaEventSynchronize(e1));
                float t = 0.f;
                CUDA_TRY(cudaEventElapsedTime(&t, e0, e1));
                ms = t / reps;
                if (ms < best) {
                    best = ms;
                    best_v = v;
                }
            }
        }
        if (ms_out) ms_out[v] = ms;
    }
    if (ms_out) ms_out[0] = best;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    A->variant = best_v;
    if (chosen) *chosen = best_v;
    return CRSD_OK;
}

// Build-time autotuning: the row-segment height changes the layout itself
// (P:L351-361), so every candidate is built, its kernel variant autotuned on
// scratch vectors, and the fastest handle kept (one candidate resident at a
// time besides the best so far).
crsd_status_t crsd_create_autotuned(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row, const int64_t *col,
                                    const void *val, crsd_dtype_t dtype, const crsd_opts_t *opts,
                                    const int32_t *mrows_cand, int32_t ncand, int32_t reps, crsd_matrix_t *out,
                                    double *ms_out) {
    if (!out) return fail(CRSD_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    crsd_opts_t o;
    if (opts) o = *opts;
    else crsd_opts_init(&o);
    if (o.flags & CRSD_HOST_ONLY) return fail(CRSD_ERR_UNSUPPORTED, "autotuning needs a GPU handle");
    if (o.row_begin != 0 || (o.row_end != 0 && o.row_end != nrows))
        return fail(CRSD_ERR_UNSUPPORTED, "autotuning is for one-GPU (non-partitioned) handles");
    const int32_t dflt[] = {0};
    if (!mrows_cand || ncand <= 0) {
        mrows_cand = dflt;
        ncand = 1;
    }
    const size_t es = dtype == CRSD_R64F ? 8 : 4;
    void *x = nullptr, *y = nullptr;
    crsd_matrix_t best = nullptr;
    double best_ms = 1e300;
    crsd_status_t st = CRSD_OK;
    for (int32_t c = 0; c < ncand; ++c) {
        crsd_opts_t oc = o;
        oc.mrows = mrows_cand[c];
        crsd_matrix_t A = nullptr;
        crsd_status_t sc = crsd_create_from_coo(nrows, ncols, nnz, row, col, val, dtype, &oc, &A);
        if (ms_out) ms_out[c] = -1.0;
        if (sc) continue;  // this candidate is not valid for the GPU path (e.g. mrows alignment)
        if (!x) {
            cudaError_t e1 = cudaMalloc(&x, es * (size_t)ncols), e2 = cudaMalloc(&y, es * (size_t)nrows);
            if (e1 != cudaSuccess || e2 != cudaSuccess) {
                crsd_destroy(A);
                st = fail(CRSD_ERR_ALLOC, "autotune scratch vectors");
                break;
            }
            cudaMemset(x, 0, es * (size_t)ncols);  // values do not change the timing
        }
        double ms[5];
        int32_t chosen = 0;
        sc = crsd_autotune(A, x, y, reps, ms, &chosen, nullptr);
        if (sc) {
            crsd_destroy(A);
            continue;
        }
        if (ms_out) ms_out[c] = ms[0];
        if (ms[0] < best_ms) {
            if (best) crsd_destroy(best);
            best = A;
            best_ms = ms[0];
        } else {
            crsd_destroy(A);
        }
    }
    if (x) cudaFree(x);
    if (y) cudaFree(y);
    if (st) {
        if (best) crsd_destroy(best);
        return st;
    }
    if (!best) return fail(CRSD_ERR_UNSUPPORTED, "no mrows candidate is valid for the GPU path");
    *out = best;
    return CRSD_OK;
}

crsd_status_t crsd_export_paper_ell(crsd_matrix_t A, int64_t *nrows_s, int64_t *width, int64_t *rowno,
                                    int64_t *colval, void *val) {
    if (!A) return fail(CRSD_ERR_INVALID_ARG, "A is NULL");
    const HostCRSD &H = A->H;
    if (!H.paper_ell) return fail(CRSD_ERR_UNSUPPORTED, "handle built without CRSD_PAPER_ELL");
    if (nrows_s) *nrows_s = H.ell_nrows;
    if (width) *width = H.ell_width;
    if (rowno)
        for (int64_t i = 0; i < H.ell_nrows; ++i) rowno[i] = H.ell_rowno[i] + H.row_begin;
    if (colval && !H.ell_col.empty()) std::memcpy(colval, H.ell_col.data(), H.ell_col.size() * 8);
    if (val && !H.ell_val.empty()) std::memcpy(val, H.ell_val.data(), H.ell_val.size());
    return CRSD_OK;
}

crsd_status_t crsd_last_launch_count(crsd_matrix_t A, int32_t *count) {
    if (!A || !count) return fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    *count = A->last_launches;
    return CRSD_OK;
}

crsd_status_t crsd_dist_x_layout(crsd_matrix_t A, int64_t *halo_lo, int64_t *n_local, int64_t *halo_hi) {
    if (!A) return fail(CRSD_ERR_INVALID_ARG, "A is NULL");
    if (halo_lo) *halo_lo = A->halo_lo;
    if (n_local) *n_local = A->H.n_local;
    if (halo_hi) *halo_hi = A->halo_hi;
    return CRSD_OK;
}

crsd_status_t crsd_dist_ranges(crsd_matrix_t A, int64_t *r4) {
    if (!A || !r4) return fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    r4[0] = A->H.row_begin;
    r4[1] = A->H.row_end;
    r4[2] = A->halo_lo_valid;
    r4[3] = A->halo_hi_valid;
    return CRSD_OK;
}

crsd_status_t crsd_partition_rows(int64_t nrows, int32_t mrows, int world, const double *weights, int64_t *bounds) {
    if (nrows <= 0 || mrows <= 0 || world <= 0 || !bounds) return fail(CRSD_ERR_INVALID_ARG, "bad argument");
    const int64_t nseg = (nrows + mrows - 1) / mrows;
    if (world > nseg)
        return fail(CRSD_ERR_INVALID_ARG, "crsd_partition_rows: " + std::to_string(world) + " ranks but only " +
                                              std::to_string(nseg) + " row segments (every rank needs one)");
    // per-segment weight prefix; cut where the prefix crosses k/world of the total
    std::vector<double> pre(nseg + 1, 0.0);
    for (int64_t s = 0; s < nseg; ++s) {
        double w = 0.0;
        const int64_t r1 = std::min<int64_t>(nrows, (s + 1) * mrows);
        if (weights) {
            for (int64_t r = s * mrows; r < r1; ++r) w += weights[r];
        } else {
            w = double(r1 - s * mrows);
        }
        pre[s + 1] = pre[s] + w;
    }
    bounds[0] = 0;
    int64_t s = 0;
    for (int k = 1; k < world; ++k) {
        const double target = pre[nseg] * k / world;
        while (s < nseg && pre[s + 1] <= target) ++s;
        // choose the nearer boundary
        int64_t cut = s;
        if (s < nseg && (pre[s + 1] - target) < (target - pre[s])) cut = s + 1;
        // every rank keeps at least one segment: after the previous cut, and
        // early enough that each remaining rank still gets one
        const int64_t prev = (bounds[k - 1] + mrows - 1) / mrows;
        cut = std::max(cut, prev + 1);
        cut = std::min<int64_t>(cut, nseg - (world - k));
        bounds[k] = std::min<int64_t>(nrows, cut * mrows);
    }
    bounds[world] = nrows;
    return CRSD_OK;
}

}  // extern "C"
