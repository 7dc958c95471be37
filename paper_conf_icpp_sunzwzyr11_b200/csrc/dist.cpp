// Row-partitioned multi-GPU CRSD SpMV (BASELINE.json north_star (3); not in
// the paper, which is single-GPU).
//
// Each rank owns rows [row_begin, row_end) of a square matrix and the same
// range of x. Rows are independent given x (one work-item per
// row), so the only exchange is the x halo: rank r needs x[row_begin -
// halo_lo, row_begin) and x[row_end, row_end + halo_hi). The halo moves with
// NCCL send/recv on a comm stream, received straight into the pads of the
// caller's padded x buffer, while the interior segments (whose x windows and
// scatter columns stay inside the owned range) run on the compute stream;
// the boundary segments run after the halo event. y stays row-distributed:
// no reduction.
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include "crsd_handle.h"
#include "crsd_internal.h"

#include "crsd_comm.h"

namespace {
crsd_status_t nccl_fail(ncclResult_t r, const char *what) {
    return crsd::fail(CRSD_ERR_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}
crsd_status_t cu_fail(cudaError_t e, const char *what) {
    return crsd::fail(CRSD_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}
}  // namespace

#define NCCL_TRY(expr)                                        \
    do {                                                      \
        ncclResult_t _r = (expr);                             \
        if (_r != ncclSuccess) return nccl_fail(_r, #expr); \
    } while (0)
#define CU_TRY(expr)                                        \
    do {                                                    \
        cudaError_t _e = (expr);                            \
        if (_e != cudaSuccess) return cu_fail(_e, #expr); \
    } while (0)

extern "C" {

crsd_status_t crsd_comm_unique_id(void *id128) {
    if (!id128) return crsd::fail(CRSD_ERR_INVALID_ARG, "id is NULL");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId must be 128 bytes");
    NCCL_TRY(ncclGetUniqueId((ncclUniqueId *)id128));
    return CRSD_OK;
}

crsd_status_t crsd_comm_init_rank(const void *id128, int rank, int world, int device, crsd_comm_t *out) {
    if (!id128 || !out || world <= 0 || rank < 0 || rank >= world)
        return crsd::fail(CRSD_ERR_INVALID_ARG, "bad communicator arguments");
    *out = nullptr;
    CU_TRY(cudaSetDevice(device));
    crsd_comm_s *c = new crsd_comm_s();
    c->rank = rank;
    c->world = world;
    c->device = device;
    ncclUniqueId id;
    std::memcpy(&id, id128, sizeof(id));
    ncclResult_t r = ncclCommInitRank(&c->comm, world, id, rank);
    if (r != ncclSuccess) {
        delete c;
        return nccl_fail(r, "ncclCommInitRank");
    }
    CU_TRY(cudaStreamCreateWithFlags(&c->cs, cudaStreamNonBlocking));
    CU_TRY(cudaEventCreateWithFlags(&c->ev_x, cudaEventDisableTiming));
    CU_TRY(cudaEventCreateWithFlags(&c->ev_halo, cudaEventDisableTiming));
    *out = c;
    return CRSD_OK;
}

crsd_status_t crsd_comm_destroy(crsd_comm_t c) {
    if (!c) return CRSD_OK;
    cudaSetDevice(c->device);
    if (c->cs) cudaStreamSynchronize(c->cs);
    if (c->comm) ncclCommDestroy(c->comm);
    if (c->ev_x) cudaEventDestroy(c->ev_x);
    if (c->ev_halo) cudaEventDestroy(c->ev_halo);
    if (c->cs) cudaStreamDestroy(c->cs);
    delete c;
    return CRSD_OK;
}

crsd_status_t crsd_dist_plan(int world, int rank, const int64_t *rg, int64_t *recv_peer, int64_t *recv_begin,
                             int64_t *recv_count, int64_t *nrecv, int64_t *send_peer, int64_t *send_begin,
                             int64_t *send_count, int64_t *nsend) {
    if (world <= 0 || rank < 0 || rank >= world || !rg || !nrecv || !nsend)
        return crsd::fail(CRSD_ERR_INVALID_ARG, "bad plan arguments");
    for (int q = 0; q < world; ++q) {
        if (rg[4 * q] >= rg[4 * q + 1]) return crsd::fail(CRSD_ERR_INVALID_ARG, "empty row range");
        if (q > 0 && rg[4 * q] != rg[4 * (q - 1) + 1])
            return crsd::fail(CRSD_ERR_INVALID_ARG, "row ranges not contiguous");
        if (rg[4 * q + 2] < 0 || rg[4 * q + 3] < 0) return crsd::fail(CRSD_ERR_INVALID_ARG, "negative halo");
    }
    if (rg[0] != 0) return crsd::fail(CRSD_ERR_INVALID_ARG, "row ranges must start at 0");
    auto need = [&](int q, int side, int64_t &a, int64_t &b) {
        if (side == 0) {
            a = rg[4 * q] - rg[4 * q + 2];
            b = rg[4 * q];
        } else {
            a = rg[4 * q + 1];
            b = rg[4 * q + 1] + rg[4 * q + 3];
        }
    };
    int64_t nr = 0, nsd = 0;
    for (int q = 0; q < world; ++q) {
        if (q == rank) continue;
        // what I receive from q: my needs intersected with q's rows
        for (int side = 0; side < 2; ++side) {
            int64_t a, b;
            need(rank, side, a, b);
            a = std::max(a, rg[4 * q]);
            b = std::min(b, rg[4 * q + 1]);
            if (a < b) {
                if (recv_peer) recv_peer[nr] = q;
                if (recv_begin) recv_begin[nr] = a;
                if (recv_count) recv_count[nr] = b - a;
                ++nr;
            }
        }
        // what I send to q: q's needs intersected with my rows
        for (int side = 0; side < 2; ++side) {
            int64_t a, b;
            need(q, side, a, b);
            a = std::max(a, rg[4 * rank]);
            b = std::min(b, rg[4 * rank + 1]);
            if (a < b) {
                if (send_peer) send_peer[nsd] = q;
                if (send_begin) send_begin[nsd] = a;
                if (send_count) send_count[nsd] = b - a;
                ++nsd;
            }
        }
    }
    *nrecv = nr;
    *nsend = nsd;
    return CRSD_OK;
}

crsd_status_t crsd_dist_bind(crsd_matrix_t A, crsd_comm_t c, void *stream) {
    if (!A || !c) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    if (A->host_only) return crsd::fail(CRSD_ERR_UNSUPPORTED, "host-only handle");
    CU_TRY(cudaSetDevice(A->device));
    const int W = c->world;
    int64_t mine[4] = {A->H.row_begin, A->H.row_end, A->halo_lo_valid, A->halo_hi_valid};
    int64_t *d = nullptr;
    CU_TRY(cudaMalloc(&d, sizeof(int64_t) * 4 * (W + 1)));
    CU_TRY(cudaMemcpy(d, mine, sizeof(mine), cudaMemcpyHostToDevice));
    cudaStream_t s = (cudaStream_t)stream;
    ncclResult_t r = ncclAllGather(d, d + 4, 4, ncclInt64, c->comm, s);
    std::vector<int64_t> all(4 * W);
    cudaError_t e = cudaStreamSynchronize(s);
    if (r == ncclSuccess && e == cudaSuccess)
        e = cudaMemcpy(all.data(), d + 4, sizeof(int64_t) * 4 * W, cudaMemcpyDeviceToHost);
    cudaFree(d);
    if (r != ncclSuccess) return nccl_fail(r, "ncclAllGather");
    if (e != cudaSuccess) return cu_fail(e, "allgather copy");
    std::vector<int64_t> rp(2 * W), rb(2 * W), rc(2 * W), sp(2 * W), sb(2 * W), sc(2 * W);
    int64_t nr, ns;
    crsd_status_t st = crsd_dist_plan(W, c->rank, all.data(), rp.data(), rb.data(), rc.data(), &nr, sp.data(),
                                      sb.data(), sc.data(), &ns);
    if (st) return st;
    // global column -> index into x_padded
    const int64_t origin = A->H.row_begin - A->halo_lo;
    A->recv_peer.assign(rp.begin(), rp.begin() + nr);
    A->recv_count.assign(rc.begin(), rc.begin() + nr);
    A->recv_off.resize(nr);
    for (int64_t k = 0; k < nr; ++k) A->recv_off[k] = rb[k] - origin;
    A->send_peer.assign(sp.begin(), sp.begin() + ns);
    A->send_count.assign(sc.begin(), sc.begin() + ns);
    A->send_off.resize(ns);
    for (int64_t k = 0; k < ns; ++k) A->send_off[k] = sb[k] - origin;
    A->bound = true;
    return CRSD_OK;
}

crsd_status_t crsd_spmv_dist(crsd_matrix_t A, const void *alpha, void *x_padded, const void *beta, void *y_local,
                             crsd_comm_t c, void *stream) {
    if (!A) return crsd::fail(CRSD_ERR_INVALID_ARG, "A is NULL");
    if (A->host_only) return crsd::fail(CRSD_ERR_UNSUPPORTED, "host-only handle");
    if (A->H.paper_ell) return crsd::fail(CRSD_ERR_UNSUPPORTED, "CRSD_PAPER_ELL handle: use crsd_spmv");
    if (!alpha || !beta || !x_padded || !y_local) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    if (((uintptr_t)x_padded | (uintptr_t)y_local) & 15)
        return crsd::fail(CRSD_ERR_INVALID_ARG, "x_padded and y_local must be 16-byte aligned");
    if (c && !A->bound) return crsd::fail(CRSD_ERR_INVALID_ARG, "call crsd_dist_bind first");
    CU_TRY(cudaSetDevice(A->device));
    const size_t es = A->H.elem;
    char *xp = (char *)x_padded;
    const void *xbase = xp + es * A->halo_lo;
    cudaStream_t s = (cudaStream_t)stream;
    int launches = 0;
    crsd_status_t st;
    if (c) {
        const ncclDataType_t ty = (A->H.dtype == CRSD_R64F) ? ncclFloat64 : ncclFloat32;
        CU_TRY(cudaEventRecord(c->ev_x, s));
        CU_TRY(cudaStreamWaitEvent(c->cs, c->ev_x, 0));
        NCCL_TRY(ncclGroupStart());
        for (size_t k = 0; k < A->recv_peer.size(); ++k)
            NCCL_TRY(ncclRecv(xp + es * A->recv_off[k], A->recv_count[k], ty, (int)A->recv_peer[k], c->comm, c->cs));
        for (size_t k = 0; k < A->send_peer.size(); ++k)
            NCCL_TRY(ncclSend(xp + es * A->send_off[k], A->send_count[k], ty, (int)A->send_peer[k], c->comm, c->cs));
        NCCL_TRY(ncclGroupEnd());
        CU_TRY(cudaEventRecord(c->ev_halo, c->cs));
    }
    st = crsd::run_lists(A, alpha, xbase, beta, y_local, (const int32_t *)A->d_list_interior, 0,
                         (int64_t)A->list_interior.size(), stream, launches);
    if (st) return st;
    if (c) CU_TRY(cudaStreamWaitEvent(s, c->ev_halo, 0));
    st = crsd::run_lists(A, alpha, xbase, beta, y_local, (const int32_t *)A->d_list_boundary, 0,
                         (int64_t)A->list_boundary.size(), stream, launches);
    A->last_launches = launches;
    return st;
}

}  // extern "C"
