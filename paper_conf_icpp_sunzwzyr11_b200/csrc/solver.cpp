// crsd_cg: conjugate gradient on a CRSD matrix, one GPU or row-partitioned
// over NCCL. The algorithm is the textbook one
// (Hestenes & Stiefel; Saad Alg. 6.18, the paper's reference [2]),
// step for step as in oracle/cg_ref.py; the device kernels are in cg.cu.
//
// One GPU: a batch of `check_every` steps (SpMV + three vector kernels each)
// is captured once into a CUDA graph and replayed; scalars never leave the
// device and the stopping test runs on the device after every step, so the
// host polls one flag per batch. Multi-GPU: every step runs crsd_spmv_dist
// (halo exchange overlapped with interior segments) and the two dot products
// are NCCL allreduces of one (two at start) fp64 scalars in device memory.
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

#include "crsd_cg.h"
#include "crsd_comm.h"
#include "crsd_handle.h"
#include "crsd_internal.h"

using namespace crsd;

namespace {

crsd_status_t cu_fail(cudaError_t e, const char *what) {
    return fail(CRSD_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

#define CU_TRY(expr)                                        \
    do {                                                    \
        cudaError_t _e = (expr);                            \
        if (_e != cudaSuccess) return cu_fail(_e, #expr); \
    } while (0)
#define NC_TRY(expr)                                                                                     \
    do {                                                                                                 \
        ncclResult_t _r = (expr);                                                                        \
        if (_r != ncclSuccess) return fail(CRSD_ERR_NCCL, std::string(#expr) + ": " + ncclGetErrorString(_r)); \
    } while (0)
#define ST_TRY(expr)                    \
    do {                                \
        crsd_status_t _s = (expr);      \
        if (_s != CRSD_OK) return _s;   \
    } while (0)

inline int64_t up256(int64_t b) { return (b + 255) / 256 * 256; }

struct Ws {
    CgState *st;
    double *partials, *hist;
    char *r, *q, *p_pad;  // p_pad: halo_lo + n + halo_hi elements
};

crsd_status_t workspace(crsd_matrix_s *A, int64_t max_iter, int grid, Ws &w) {
    const int64_t es = A->H.elem, n = A->H.n_local;
    const int64_t npad = A->halo_lo + n + A->halo_hi;
    const int64_t o_part = up256(sizeof(CgState));
    const int64_t o_hist = o_part + up256(8 * (int64_t)grid);
    const int64_t o_r = o_hist + up256(8 * (max_iter + 1));
    const int64_t o_q = o_r + up256(es * n);
    const int64_t o_p = o_q + up256(es * n);
    const int64_t total = o_p + up256(es * npad);
    if (total > A->cg_bytes) {
        if (A->d_cg) {
            cudaFree(A->d_cg);
            A->device_bytes -= A->cg_bytes;
        }
        A->d_cg = nullptr;
        A->cg_bytes = 0;
        cudaError_t e = cudaMalloc(&A->d_cg, total);
        if (e != cudaSuccess) {
            A->d_cg = nullptr;
            return fail(e == cudaErrorMemoryAllocation ? CRSD_ERR_ALLOC : CRSD_ERR_CUDA,
                        "CG workspace cudaMalloc(" + std::to_string(total) + "): " + cudaGetErrorString(e));
        }
        A->cg_bytes = total;
        A->device_bytes += total;
        CU_TRY(cudaMemset(A->d_cg, 0, total));  // counters, halo pads
    }
    char *b = (char *)A->d_cg;
    w.st = (CgState *)b;
    w.partials = (double *)(b + o_part);
    w.hist = (double *)(b + o_hist);
    w.r = b + o_r;
    w.q = b + o_q;
    w.p_pad = b + o_p;
    return CRSD_OK;
}

template <typename T>
crsd_status_t cg_impl(crsd_matrix_s *A, const T *b, T *x, int32_t max_iter, double rtol, int32_t check_every,
                      crsd_comm_s *comm, double *rr_history, crsd_cg_result_t *res, cudaStream_t user) {
    const int64_t n = A->H.n_local, es = sizeof(T), nseg = A->H.nseg;
    const int grid = cg_grid(A->sm_count);
    Ws w;
    ST_TRY(workspace(A, max_iter, grid, w));
    if (!A->cg_stream) {
        cudaStream_t s;
        cudaEvent_t e1, e2;
        CU_TRY(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
        CU_TRY(cudaEventCreateWithFlags(&e1, cudaEventDisableTiming));
        CU_TRY(cudaEventCreateWithFlags(&e2, cudaEventDisableTiming));
        A->cg_stream = s;
        A->cg_ev_in = e1;
        A->cg_ev_out = e2;
    }
    // all work on the handle's stream, ordered after / before the caller's
    cudaStream_t s = (cudaStream_t)A->cg_stream;
    CU_TRY(cudaEventRecord((cudaEvent_t)A->cg_ev_in, user));
    CU_TRY(cudaStreamWaitEvent(s, (cudaEvent_t)A->cg_ev_in, 0));

    T *r = (T *)w.r, *q = (T *)w.q;
    // peer-memory transport: p lives in the handle's crsd_dist_x_alloc
    // buffer, so every halo moves as one-sided puts into the neighbours'
    // pads (collective: every rank runs crsd_cg)
    if (comm && comm->kind == crsd_comm_s::P2P && comm->world > 1) {
        const crsd_matrix_s::DirectX *d = nullptr;
        for (const crsd_matrix_s::DirectX &e : A->dx)
            if (e.purpose == 1) d = &e;
        if (d && d->comm != comm)
            return fail(CRSD_ERR_INVALID_ARG, "the handle's CG direct buffer belongs to another communicator");
        void *pp = d ? d->own : nullptr;
        if (!d) ST_TRY(dist_x_alloc(A, comm, 1, &pp));
        w.p_pad = (char *)pp;
    }
    T *p_own = (T *)w.p_pad + A->halo_lo;
    int launches = 0;
    auto spmv = [&](T al, T be, T *y) -> crsd_status_t {
        if (comm) {
            // boundary placement as crsd_spmv_dist (the handle's
            // CRSD_TUNE_DIST_BOUNDARY_SERIAL). Under MPS (ranks sharing one
            // GPU) the CG is bimodal: one run favoured serial 2-3x, the next
            // concurrent 2x (profiles/r01_ab_boundary_cg_*, r01_ab_cg_*), so the
            // default follows the SpMV measurement and the no-serial-tail argument.
            ST_TRY(spmv_dist_impl(A, &al, w.p_pad, &be, y, comm, s, -1));
            launches += A->last_launches;
            return CRSD_OK;
        }
        return run_lists(A, &al, p_own, &be, y, nullptr, 0, nseg, s, launches);
    };
    auto kerr = [&](int e, const char *what) -> crsd_status_t {
        if (e) return cu_fail((cudaError_t)e, what);
        ++launches;
        return CRSD_OK;
    };

    // state
    CgState h;
    std::memset(&h, 0, sizeof(h));
    h.rtol = rtol;
    h.max_iter = max_iter;
    h.hist_cap = max_iter;
    h.hist = w.hist;
    h.partials = w.partials;
    CU_TRY(cudaMemcpyAsync(w.st, &h, sizeof(h), cudaMemcpyHostToDevice, s));

    // r_0 = b - A x_0, p_0 = r_0, rr_0 = (r_0, r_0), bb = (b, b)
    CU_TRY(cudaMemcpyAsync(p_own, x, es * n, cudaMemcpyDeviceToDevice, s));
    CU_TRY(cudaMemcpyAsync(r, b, es * n, cudaMemcpyDeviceToDevice, s));
    ST_TRY(spmv(T(-1), T(1), r));
    CU_TRY(cudaMemcpyAsync(p_own, r, es * n, cudaMemcpyDeviceToDevice, s));
    ST_TRY(kerr(cg_launch_dot<T>(r, r, n, w.st, CG_RR, false, grid, s), "cg_dot(r,r)"));
    ST_TRY(kerr(cg_launch_dot<T>(b, b, n, w.st, CG_BB, false, grid, s), "cg_dot(b,b)"));
    if (comm) ST_TRY(comm_allreduce_f64(comm, w.st->red + CG_RR, 2, s));
    ST_TRY(kerr(cg_launch_init(w.st, s), "cg_init"));

    // (p, q) is a separate kernel. Fusing it into the SpMV epilogue (round 1,
    // removed) saved two vector passes but lengthened every SpMV CTA's life
    // (fewer bytes in flight): C2 f64 0.417 vs 0.407 ms/step, f32 equal
    // (profiles/r01_cg_ab.jsonl).
    auto step = [&]() -> crsd_status_t {
        ST_TRY(spmv(T(1), T(0), q));  // q = A p
        ST_TRY(kerr(cg_launch_dot<T>(p_own, q, n, w.st, CG_PQ, true, grid, s), "cg_dot(p,q)"));
        if (comm) ST_TRY(comm_allreduce_f64(comm, w.st->red + CG_PQ, 1, s));
        ST_TRY(kerr(cg_launch_update<T>(r, q, n, w.st, grid, s), "cg_update"));
        if (comm) ST_TRY(comm_allreduce_f64(comm, w.st->red + CG_RR, 1, s));
        ST_TRY(kerr(cg_launch_pupdate<T>(p_own, r, x, n, w.st, grid, s), "cg_pupdate"));
        return CRSD_OK;
    };

    int32_t done = 0;
    CU_TRY(cudaMemcpyAsync(&done, &w.st->done, sizeof(done), cudaMemcpyDeviceToHost, s));
    CU_TRY(cudaStreamSynchronize(s));
    const int32_t batch = std::max<int32_t>(1, std::min<int32_t>(check_every, std::max<int32_t>(max_iter, 1)));
    cudaGraphExec_t exec = nullptr;
    int graph_launches = 0;
    for (int64_t issued = 0; !done && issued < max_iter; issued += batch) {
        // One batch of steps as a CUDA graph: one GPU, or the peer-memory
        // transport (its exchange and allreduce kernels keep their epochs on
        // the device, so a replay is a new exchange). NCCL calls are issued
        // directly.
        if (!comm || comm->kind == crsd_comm_s::P2P) {
            if (!exec) {
                const int l0 = launches;
                cudaGraph_t g;
                CU_TRY(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
                crsd_status_t st = CRSD_OK;
                for (int32_t k = 0; k < batch && !st; ++k) st = step();
                cudaError_t ce = cudaStreamEndCapture(s, &g);
                if (st) {
                    if (ce == cudaSuccess) cudaGraphDestroy(g);
                    return st;
                }
                CU_TRY(ce);
                cudaError_t ie = cudaGraphInstantiate(&exec, g, 0);
                cudaGraphDestroy(g);
                CU_TRY(ie);
                graph_launches = launches - l0;
                launches = l0;
            }
            CU_TRY(cudaGraphLaunch(exec, s));
            launches += graph_launches;
        } else {
            for (int32_t k = 0; k < batch; ++k) ST_TRY(step());
        }
        CU_TRY(cudaMemcpyAsync(&done, &w.st->done, sizeof(done), cudaMemcpyDeviceToHost, s));
        CU_TRY(cudaStreamSynchronize(s));
    }
    if (exec) cudaGraphExecDestroy(exec);

    CU_TRY(cudaMemcpyAsync(&h, w.st, sizeof(h), cudaMemcpyDeviceToHost, s));
    CU_TRY(cudaStreamSynchronize(s));
    if (rr_history) CU_TRY(cudaMemcpy(rr_history, w.hist, sizeof(double) * (h.it + 1), cudaMemcpyDeviceToHost));
    CU_TRY(cudaEventRecord((cudaEvent_t)A->cg_ev_out, s));
    CU_TRY(cudaStreamWaitEvent(user, (cudaEvent_t)A->cg_ev_out, 0));
    if (res) {
        res->iterations = (int32_t)h.it;
        res->converged = h.rr <= h.tol2 ? 1 : 0;
        res->rr0 = 0.0;
        res->rr = h.rr;
        res->bb = h.bb;
        res->launches = launches;
    }
    if (res) {
        double rr0 = 0.0;
        CU_TRY(cudaMemcpy(&rr0, w.hist, sizeof(double), cudaMemcpyDeviceToHost));
        res->rr0 = rr0;
    }
    A->last_launches = launches;
    return CRSD_OK;
}

}  // namespace

extern "C" crsd_status_t crsd_cg(crsd_matrix_t A, const void *b, void *x, int32_t max_iter, double rtol,
                                 int32_t check_every, crsd_comm_t comm, double *rr_history, crsd_cg_result_t *res,
                                 void *stream) {
    NvtxRange nv("crsd_cg");
    if (!A) return fail(CRSD_ERR_INVALID_ARG, "A is NULL");
    if (A->host_only) return fail(CRSD_ERR_UNSUPPORTED, "host-only handle");
    if (!b || !x) return fail(CRSD_ERR_INVALID_ARG, "b and x must not be NULL");
    if (((uintptr_t)b | (uintptr_t)x) & 15) return fail(CRSD_ERR_INVALID_ARG, "b and x must be 16-byte aligned");
    if (b == x) return fail(CRSD_ERR_INVALID_ARG, "b and x must not alias");
    if (max_iter < 0 || !(rtol >= 0.0)) return fail(CRSD_ERR_INVALID_ARG, "max_iter must be >= 0 and rtol >= 0");
    if (A->H.nrows != A->H.ncols) return fail(CRSD_ERR_UNSUPPORTED, "CG needs a square matrix");
    if (A->H.paper_ell) return fail(CRSD_ERR_UNSUPPORTED, "CRSD_PAPER_ELL handle: CG needs y = alpha*A*x + beta*y");
    if (A->H.partitioned && !comm) return fail(CRSD_ERR_INVALID_ARG, "row-partitioned handle: pass its communicator");
    if (comm && !A->bound) return fail(CRSD_ERR_INVALID_ARG, "call crsd_dist_bind first");
    if (check_every <= 0) check_every = 16;
    CU_TRY(cudaSetDevice(A->device));
    if (A->H.dtype == CRSD_R64F)
        return cg_impl<double>(A, (const double *)b, (double *)x, max_iter, rtol, check_every, comm, rr_history, res,
                               (cudaStream_t)stream);
    return cg_impl<float>(A, (const float *)b, (float *)x, max_iter, rtol, check_every, comm, rr_history, res,
                          (cudaStream_t)stream);
}
