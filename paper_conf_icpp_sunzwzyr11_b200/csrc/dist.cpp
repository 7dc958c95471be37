// Row-partitioned multi-GPU CRSD SpMV (BASELINE.json north_star (3); not in
// the paper, which is single-GPU).
//
// Each rank owns rows [row_begin, row_end) of a square matrix and the same
// range of x. Rows are independent given x (one work-item per
// row), so the only exchange is the x halo: rank r needs x[row_begin -
// halo_lo, row_begin) and x[row_end, row_end + halo_hi). The halo moves on
// a comm stream, received straight into the pads of the caller's padded x
// buffer, while the interior segments (whose x windows and scatter columns
// stay inside the owned range) run on the compute stream; the boundary
// segments run on the comm stream behind the exchange, concurrently with the
// interior, and the compute stream joins at the end. y stays
// row-distributed: no reduction.
//
// Two transports behind crsd_comm_t: NCCL (grouped send/recv), or the
// library's own peer-memory kernels (p2p.cu) over CUDA-IPC-mapped symmetric
// regions — loads over NVLink/NVSwitch from the neighbour's mailbox straight
// into the pads, flag handshakes in peer memory, no NCCL on the data path.
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cstddef>
#include <cstdlib>
#include <cstring>
#include <chrono>
#include <string>
#include <thread>
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
#define ST_TRY(expr)                  \
    do {                              \
        crsd_status_t _s = (expr);    \
        if (_s != CRSD_OK) return _s; \
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
    int prio_lo = 0, prio_hi = 0;
    CU_TRY(cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi));
    CU_TRY(cudaStreamCreateWithPriority(&c->cs, cudaStreamNonBlocking, prio_hi));
    CU_TRY(cudaEventCreateWithFlags(&c->ev_x, cudaEventDisableTiming));
    CU_TRY(cudaEventCreateWithFlags(&c->ev_halo, cudaEventDisableTiming));
    *out = c;
    return CRSD_OK;
}

crsd_status_t crsd_comm_destroy(crsd_comm_t c) {
    if (!c) return CRSD_OK;
    cudaSetDevice(c->device);
    if (c->cs) cudaStreamSynchronize(c->cs);
    if (c->kind == crsd_comm_s::P2P && c->opened && c->world > 1) {
        // Collective close (every rank calls crsd_comm_destroy): a fast rank
        // must not free (or let the allocator reuse) its region while a
        // slower peer's last exchange still reads its mailbox or writes its
        // flags. All this rank's work on the device is finished first; then
        // every rank announces "done with your region" to every peer and
        // waits (bounded) for all peers' announcements before unmapping.
        cudaDeviceSynchronize();
        crsd::P2PReduce R{};
        R.local = (crsd::P2PFlags *)c->sym;
        R.rank = c->rank;
        R.world = c->world;
        R.timeout_ns = c->timeout_ns;
        for (int q = 0; q < c->world; ++q) R.peer_flags[q] = (crsd::P2PFlags *)c->peer_sym[q];
        if (crsd::p2p_launch_close(R, 1, c->cs) == 0) cudaStreamSynchronize(c->cs);
    }
    if (c->comm) ncclCommDestroy(c->comm);
    for (void *p : c->peer_sym)
        if (p) cudaIpcCloseMemHandle(p);
    if (c->sym) cudaFree(c->sym);
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

crsd_status_t crsd_comm_init_p2p(int rank, int world, int device, int64_t mailbox_bytes, void *ipc_handle64,
                                 crsd_comm_t *out) {
    if (!out || !ipc_handle64 || world <= 0 || world > crsd::P2P_MAX_WORLD || rank < 0 || rank >= world ||
        mailbox_bytes < 0)
        return crsd::fail(CRSD_ERR_INVALID_ARG, "bad peer-memory communicator arguments");
    *out = nullptr;
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "cudaIpcMemHandle_t must be 64 bytes");
    CU_TRY(cudaSetDevice(device));
    crsd_comm_s *c = new crsd_comm_s();
    c->kind = crsd_comm_s::P2P;
    c->rank = rank;
    c->world = world;
    c->device = device;
    c->cap = (mailbox_bytes + 255) / 256 * 256;
    c->peer_sym.assign(world, nullptr);
    c->peer_cap.assign(world, 0);
    c->peer_same_gpu.assign(world, 0);
    if (const char *t = getenv("CRSD_P2P_TIMEOUT_S")) {
        const double sec = atof(t);
        if (sec > 0) c->timeout_ns = (uint64_t)(sec * 1e9);
    }
    const size_t bytes = crsd::P2P_FLAGS_BYTES + 2 * c->cap;
    cudaError_t e = cudaMalloc(&c->sym, bytes);
    if (e == cudaSuccess) e = cudaMemset(c->sym, 0, crsd::P2P_FLAGS_BYTES);
    if (e == cudaSuccess)
        e = cudaMemcpy((char *)c->sym + offsetof(crsd::P2PFlags, cap), &c->cap, sizeof(int64_t),
                       cudaMemcpyHostToDevice);
    cudaDeviceProp prop;
    if (e == cudaSuccess) e = cudaGetDeviceProperties(&prop, device);
    if (e == cudaSuccess)
        e = cudaMemcpy((char *)c->sym + offsetof(crsd::P2PFlags, dev_uuid), &prop.uuid, 16, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaIpcGetMemHandle((cudaIpcMemHandle_t *)ipc_handle64, c->sym);
    int prio_lo = 0, prio_hi = 0;
    if (e == cudaSuccess) e = cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
    if (e == cudaSuccess) e = cudaStreamCreateWithPriority(&c->cs, cudaStreamNonBlocking, prio_hi);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_x, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_halo, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        crsd_comm_destroy(c);
        return cu_fail(e, "peer-memory communicator setup");
    }
    *out = c;
    return CRSD_OK;
}

crsd_status_t crsd_comm_p2p_open(crsd_comm_t c, const void *ipc_handles) {
    if (!c || !ipc_handles) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    if (c->kind != crsd_comm_s::P2P) return crsd::fail(CRSD_ERR_INVALID_ARG, "not a peer-memory communicator");
    if (c->opened) return crsd::fail(CRSD_ERR_INVALID_ARG, "communicator already opened");
    CU_TRY(cudaSetDevice(c->device));
    for (int q = 0; q < c->world; ++q) {
        if (q == c->rank) continue;
        cudaIpcMemHandle_t h;
        std::memcpy(&h, (const char *)ipc_handles + 64 * q, 64);
        void *p = nullptr;
        CU_TRY(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
        c->peer_sym[q] = p;
        // the peer wrote its capacity before exporting the handle
        CU_TRY(cudaMemcpy(&c->peer_cap[q], (char *)p + offsetof(crsd::P2PFlags, cap), sizeof(int64_t),
                          cudaMemcpyDeviceToHost));
        uint8_t uq[16], um[16];
        CU_TRY(cudaMemcpy(uq, (char *)p + offsetof(crsd::P2PFlags, dev_uuid), 16, cudaMemcpyDeviceToHost));
        CU_TRY(cudaMemcpy(um, (char *)c->sym + offsetof(crsd::P2PFlags, dev_uuid), 16, cudaMemcpyDeviceToHost));
        c->peer_same_gpu[q] = std::memcmp(uq, um, 16) == 0;
    }
    c->opened = true;
    return CRSD_OK;
}

crsd_status_t crsd_comm_error(crsd_comm_t c, int32_t *err) {
    if (!c || !err) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    *err = 0;
    if (c->kind != crsd_comm_s::P2P) return CRSD_OK;
    CU_TRY(cudaSetDevice(c->device));
    uint32_t v = 0;
    CU_TRY(cudaMemcpy(&v, (char *)c->sym + offsetof(crsd::P2PFlags, err), sizeof(v), cudaMemcpyDeviceToHost));
    *err = (int32_t)v;
    if (v) c->poisoned = true;
    return CRSD_OK;
}

crsd_status_t crsd_comm_allreduce_f64(crsd_comm_t c, double *dev, int n, void *stream) {
    if (!c || !dev || n <= 0) return crsd::fail(CRSD_ERR_INVALID_ARG, "bad allreduce arguments");
    CU_TRY(cudaSetDevice(c->device));
    return crsd::comm_allreduce_f64(c, dev, n, (cudaStream_t)stream);
}

}  // extern "C"

namespace crsd {
crsd_status_t comm_allreduce_f64(crsd_comm_s *c, double *dev, int n, cudaStream_t s) {
    if (c->world == 1) return CRSD_OK;
    if (c->kind == crsd_comm_s::NCCL) {
        NCCL_TRY(ncclAllReduce(dev, dev, n, ncclFloat64, ncclSum, c->comm, s));
        return CRSD_OK;
    }
    if (!c->opened) return fail(CRSD_ERR_INVALID_ARG, "call crsd_comm_p2p_open first");
    if (c->poisoned) return fail(CRSD_ERR_CUDA, "peer-memory communicator poisoned by a timed-out wait (crsd_comm_error)");
    if (n > P2P_MAX_RED) return fail(CRSD_ERR_INVALID_ARG, "peer-memory allreduce: at most 4 values");
    P2PReduce R{};
    R.local = (P2PFlags *)c->sym;
    R.rank = c->rank;
    R.world = c->world;
    R.timeout_ns = c->timeout_ns;
    for (int q = 0; q < c->world; ++q) R.peer_flags[q] = (P2PFlags *)c->peer_sym[q];
    CU_TRY((cudaError_t)p2p_launch_allreduce(R, dev, n, s));
    return CRSD_OK;
}

namespace {
// Derive A's send/recv plan from every rank's [row_begin, row_end,
// halo_lo_valid, halo_hi_valid]; for the peer-memory transport also where
// each slice sits in the sender's mailbox (its send slices in plan order,
// 256-B aligned) and check that it fits.
crsd_status_t mailbox_layout(int W, int q, const int64_t *all, int64_t es, std::vector<int64_t> &peer,
                             std::vector<int64_t> &begin, std::vector<int64_t> &off, int64_t &total) {
    std::vector<int64_t> p(2 * W), b(2 * W), cnt(2 * W), d0(2 * W), d1(2 * W), d2(2 * W);
    int64_t n_r, n_s;
    ST_TRY(crsd_dist_plan(W, q, all, d0.data(), d1.data(), d2.data(), &n_r, p.data(), b.data(), cnt.data(), &n_s));
    peer.assign(p.begin(), p.begin() + n_s);
    begin.assign(b.begin(), b.begin() + n_s);
    off.resize(n_s);
    total = 0;
    for (int64_t k = 0; k < n_s; ++k) {
        off[k] = total;
        total += (cnt[k] * es + 255) / 256 * 256;
    }
    return CRSD_OK;
}

crsd_status_t bind_table(crsd_matrix_t A, crsd_comm_t c, const int64_t *all) {
    const int W = c->world;
    if (all[4 * c->rank] != A->H.row_begin || all[4 * c->rank + 1] != A->H.row_end)
        return fail(CRSD_ERR_INVALID_ARG, "range table does not match this handle's rows");
    std::vector<int64_t> rp(2 * W), rb(2 * W), rc(2 * W), sp(2 * W), sb(2 * W), sc(2 * W);
    int64_t nr, ns;
    ST_TRY(crsd_dist_plan(W, c->rank, all, rp.data(), rb.data(), rc.data(), &nr, sp.data(), sb.data(), sc.data(),
                          &ns));
    const int64_t es = A->H.elem;
    std::vector<int64_t> send_mb(ns), recv_mb(nr);
    if (c->kind == crsd_comm_s::P2P) {
        if (nr > P2P_MAX_ITEMS || ns > P2P_MAX_ITEMS)
            return fail(CRSD_ERR_UNSUPPORTED, "peer-memory transport: more than 16 halo slices per direction");
        std::vector<int64_t> peer, begin, off;
        int64_t total = 0;
        ST_TRY(mailbox_layout(W, c->rank, all, es, peer, begin, off, total));
        if (total > c->cap)
            return fail(CRSD_ERR_INVALID_ARG, "peer-memory mailbox too small: need " + std::to_string(total) +
                                                  " bytes per parity, have " + std::to_string(c->cap));
        for (int64_t k = 0; k < ns; ++k) send_mb[k] = off[k];
        for (int64_t k = 0; k < nr; ++k) {
            ST_TRY(mailbox_layout(W, (int)rp[k], all, es, peer, begin, off, total));
            int64_t found = -1;
            for (size_t j = 0; j < peer.size(); ++j)
                if (peer[j] == c->rank && begin[j] == rb[k]) found = off[j];
            if (found < 0) return fail(CRSD_ERR_INVALID_ARG, "inconsistent halo plan between ranks");
            recv_mb[k] = found;
        }
    }
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
    A->send_mb_off = send_mb;
    A->recv_mb_off = recv_mb;
    A->range_table.assign(all, all + 4 * W);
    A->bound = true;
    A->bound_comm = c;
    return CRSD_OK;
}

// Launch record over the distinct peers of `peers` (send or receive side).
void fill_launch(P2PLaunch &L, crsd_comm_t c, const std::vector<int64_t> &peers) {
    L.local = (P2PFlags *)c->sym;
    L.rank = c->rank;
    L.timeout_ns = c->timeout_ns;
    L.npeer = 0;
    for (int64_t q : peers) {
        bool seen = false;
        for (int k = 0; k < L.npeer; ++k) seen |= (L.peer[k] == q);
        if (!seen) {
            L.peer[L.npeer] = (int32_t)q;
            L.peer_flags[L.npeer] = (P2PFlags *)c->peer_sym[q];
            ++L.npeer;
        }
    }
}

// One halo exchange through peer memory, on the comm stream. Direct mode
// (x_padded is this handle's crsd_dist_x_alloc buffer): p2p_put stores my
// send slices straight into the receivers' pads, p2p_wait waits for my
// senders. Mailbox mode (any other x_padded): p2p_send packs my send slices
// into my mailbox and flags the receivers; p2p_recv waits for the senders'
// flags and pulls their slices into the pads. Either way p2p_release (after
// the boundary segments, release_halo) frees the pads for the next epoch.
crsd_status_t p2p_exchange(crsd_matrix_t A, crsd_comm_t c, char *xp, bool fused_recv, int &launches) {
    if (!c->opened) return fail(CRSD_ERR_INVALID_ARG, "call crsd_comm_p2p_open first");
    if (c->poisoned) return fail(CRSD_ERR_CUDA, "peer-memory communicator poisoned by a timed-out wait (crsd_comm_error)");
    const int64_t es = A->H.elem;
    // a few CTAs suffice for the halo (~2 % of a rank's bytes); every CTA of
    // p2p_recv / p2p_put holds an SM slot while it waits for the peers
    const int grid = 16;
    P2PLaunch S{}, R{};
    fill_launch(S, c, A->send_peer);
    fill_launch(R, c, A->recv_peer);
    S.nitems = (int32_t)A->send_peer.size();
    R.nitems = (int32_t)A->recv_peer.size();
    if (const crsd_matrix_s::DirectX *dx = A->find_dx(xp, c)) {
        const int W = c->world;
        for (int k = 0; k < S.nitems; ++k) {
            const int64_t q = A->send_peer[k];
            const int64_t gcol = A->send_off[k] + (A->H.row_begin - A->halo_lo);  // global column of the slice
            const int64_t q_halo_lo = (A->range_table[4 * q + 2] + 3) / 4 * 4;
            const int64_t q_origin = A->range_table[4 * q] - q_halo_lo;
            (void)W;
            S.items[k] = P2PItem{xp + es * A->send_off[k], (char *)dx->peer[q] + es * (gcol - q_origin),
                                 es * A->send_count[k], 0};
        }
        CU_TRY((cudaError_t)p2p_launch_put(S, grid, c->cs));
        ++launches;
        if (!fused_recv) {  // else the boundary kernel waits itself (crsd_jit_halo)
            CU_TRY((cudaError_t)p2p_launch_wait(R, c->cs));
            ++launches;
        }
        return CRSD_OK;
    }
    char *mb = (char *)c->sym + P2P_FLAGS_BYTES;
    for (int k = 0; k < S.nitems; ++k)
        S.items[k] = P2PItem{xp + es * A->send_off[k], mb + A->send_mb_off[k], es * A->send_count[k], c->cap};
    for (int k = 0; k < R.nitems; ++k)
        R.items[k] = P2PItem{(char *)c->peer_sym[A->recv_peer[k]] + P2P_FLAGS_BYTES + A->recv_mb_off[k],
                             xp + es * A->recv_off[k], es * A->recv_count[k], c->peer_cap[A->recv_peer[k]]};
    CU_TRY((cudaError_t)p2p_launch_send(S, grid, c->cs));
    CU_TRY((cudaError_t)p2p_launch_recv(R, grid, c->cs));
    launches += 2;
    return CRSD_OK;
}

// The receive side of a direct-mode exchange for the boundary kernel
// (crsd_jit_halo): my flags, the senders, where to release them.
void make_halo_sync(crsd_matrix_t A, crsd_comm_t c, HaloSync &h) {
    P2PFlags *me = (P2PFlags *)c->sym;
    h = HaloSync{};
    h.ready = me->ready;
    h.halo_epoch = &me->halo_epoch;
    h.counter = &me->counter[1];
    h.err = &me->err;
    h.timeout_ns = c->timeout_ns;
    h.npeer = 0;
    for (int64_t q : A->recv_peer) {
        bool seen = false;
        for (int k = 0; k < h.npeer; ++k) seen |= (h.peer[k] == q);
        if (seen) continue;
        h.peer[h.npeer] = (int32_t)q;
        h.consumed[h.npeer] = &((P2PFlags *)c->peer_sym[q])->consumed[c->rank];
        ++h.npeer;
    }
}

}  // namespace

// The boundary segments of this epoch are done with the pads: tell the senders.
crsd_status_t release_halo(crsd_matrix_t A, crsd_comm_t c) {
    P2PLaunch R{};
    fill_launch(R, c, A->recv_peer);
    CU_TRY((cudaError_t)p2p_launch_release(R, c->cs));
    return CRSD_OK;
}

// crsd_dist_x_alloc: allocate this rank's padded x (IPC-exportable), hand
// its IPC handle to every peer through the peers' flag regions (host copies
// into peer memory), wait until every peer's handle has arrived in mine
// (bounded), and map them.
crsd_status_t dist_x_alloc(crsd_matrix_t A, crsd_comm_t c, int purpose, void **out) {
    if (c->kind != crsd_comm_s::P2P || !c->opened)
        return fail(CRSD_ERR_INVALID_ARG, "crsd_dist_x_alloc needs an opened peer-memory communicator");
    if (!A->bound || A->bound_comm != c) return fail(CRSD_ERR_INVALID_ARG, "bind the handle to this communicator first");
    for (const crsd_matrix_s::DirectX &d : A->dx)
        if (d.purpose == purpose)
            return fail(CRSD_ERR_INVALID_ARG, purpose == 0 ? "the handle already has a crsd_dist_x_alloc buffer"
                                                           : "the handle already has a CG direct buffer");
    const int64_t bytes = A->H.elem * (A->halo_lo + A->H.n_local + A->halo_hi);
    void *p = nullptr;
    CU_TRY(cudaMalloc(&p, std::max<int64_t>(bytes, 256)));
    cudaError_t e = cudaMemset(p, 0, std::max<int64_t>(bytes, 256));
    cudaIpcMemHandle_t h;
    if (e == cudaSuccess) e = cudaIpcGetMemHandle(&h, p);
    if (e != cudaSuccess) {
        cudaFree(p);
        return cu_fail(e, "crsd_dist_x_alloc");
    }
    const uint64_t seq = ++c->xseq;
    const int W = c->world;
    for (int q = 0; q < W && e == cudaSuccess; ++q) {
        if (q == c->rank) continue;
        char *pf = (char *)c->peer_sym[q];
        e = cudaMemcpy(pf + offsetof(P2PFlags, xh) + 64 * c->rank, &h, 64, cudaMemcpyHostToDevice);
        const int64_t rng[4] = {A->H.row_begin, A->H.row_end, purpose, 0};
        if (e == cudaSuccess)
            e = cudaMemcpy(pf + offsetof(P2PFlags, xrange) + 32 * c->rank, rng, 32, cudaMemcpyHostToDevice);
        if (e == cudaSuccess)
            e = cudaMemcpy(pf + offsetof(P2PFlags, xseq) + 8 * c->rank, &seq, 8, cudaMemcpyHostToDevice);
    }
    std::vector<void *> peer(W, nullptr);
    const auto t0 = std::chrono::steady_clock::now();
    for (int q = 0; q < W && e == cudaSuccess; ++q) {
        if (q == c->rank) continue;
        char *mine = (char *)c->sym;
        uint64_t got = 0;
        while (e == cudaSuccess) {
            e = cudaMemcpy(&got, mine + offsetof(P2PFlags, xseq) + 8 * q, 8, cudaMemcpyDeviceToHost);
            if (got >= seq) break;
            if (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() * 1e9 > (double)c->timeout_ns) {
                for (void *m : peer)
                    if (m) cudaIpcCloseMemHandle(m);
                cudaFree(p);
                return fail(CRSD_ERR_CUDA, "crsd_dist_x_alloc: rank " + std::to_string(q) + " never published its buffer");
            }
            std::this_thread::sleep_for(std::chrono::microseconds(200));
        }
        cudaIpcMemHandle_t hq;
        int64_t rq[4] = {-1, -1, -1, 0};
        if (e == cudaSuccess) e = cudaMemcpy(&hq, mine + offsetof(P2PFlags, xh) + 64 * q, 64, cudaMemcpyDeviceToHost);
        if (e == cudaSuccess) e = cudaMemcpy(rq, mine + offsetof(P2PFlags, xrange) + 32 * q, 32, cudaMemcpyDeviceToHost);
        // the peer must have allocated for the handle this one is bound to
        // (same row block as in the range table) and for the same purpose: a
        // collective mismatch (ranks allocating for different matrices or in
        // a different order) is refused, not mapped
        if (e == cudaSuccess &&
            (rq[0] != A->range_table[4 * q] || rq[1] != A->range_table[4 * q + 1] || rq[2] != purpose)) {
            for (void *m : peer)
                if (m) cudaIpcCloseMemHandle(m);
            cudaFree(p);
            return fail(CRSD_ERR_INVALID_ARG, "crsd_dist_x_alloc: rank " + std::to_string(q) +
                                                  " allocated for a different row block (collective mismatch)");
        }
        if (e == cudaSuccess) e = cudaIpcOpenMemHandle(&peer[q], hq, cudaIpcMemLazyEnablePeerAccess);
    }
    if (e != cudaSuccess) {
        for (void *m : peer)
            if (m) cudaIpcCloseMemHandle(m);
        cudaFree(p);
        return cu_fail(e, "crsd_dist_x_alloc handshake");
    }
    crsd_matrix_s::DirectX d;
    d.own = p;
    d.peer = peer;
    d.comm = c;
    d.purpose = purpose;
    A->dx.push_back(d);
    A->device_bytes += bytes;
    if (out) *out = p;
    return CRSD_OK;
}
}  // namespace crsd

extern "C" {

crsd_status_t crsd_dist_bind(crsd_matrix_t A, crsd_comm_t c, void *stream) {
    if (!A || !c) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    if (A->host_only) return crsd::fail(CRSD_ERR_UNSUPPORTED, "host-only handle");
    if (c->kind != crsd_comm_s::NCCL)
        return crsd::fail(CRSD_ERR_INVALID_ARG, "peer-memory communicator: use crsd_dist_bind_ranges");
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
    return crsd::bind_table(A, c, all.data());
}

crsd_status_t crsd_dist_bind_ranges(crsd_matrix_t A, crsd_comm_t c, const int64_t *ranges4) {
    if (!A || !c || !ranges4) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    if (A->host_only) return crsd::fail(CRSD_ERR_UNSUPPORTED, "host-only handle");
    return crsd::bind_table(A, c, ranges4);
}

crsd_status_t crsd_dist_x_alloc(crsd_matrix_t A, crsd_comm_t c, void **x_padded) {
    if (!A || !c || !x_padded) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    *x_padded = nullptr;
    CU_TRY(cudaSetDevice(A->device));
    return crsd::dist_x_alloc(A, c, 0, x_padded);
}

crsd_status_t crsd_spmv_dist(crsd_matrix_t A, const void *alpha, void *x_padded, const void *beta, void *y_local,
                             crsd_comm_t c, void *stream) {
    return crsd::spmv_dist_impl(A, alpha, x_padded, beta, y_local, c, stream, -1);
}

}  // extern "C"

// boundary: -1 = the handle's setting (concurrent on the comm stream unless
// CRSD_TUNE_DIST_BOUNDARY_SERIAL), 0 = concurrent, 1 = serial after the interior
crsd_status_t crsd::spmv_dist_impl(crsd_matrix_t A, const void *alpha, void *x_padded, const void *beta,
                                   void *y_local, crsd_comm_t c, void *stream, int boundary) {
    crsd::NvtxRange nv("crsd_spmv_dist");
    if (!A) return crsd::fail(CRSD_ERR_INVALID_ARG, "A is NULL");
    if (A->host_only) return crsd::fail(CRSD_ERR_UNSUPPORTED, "host-only handle");
    if (A->H.paper_ell) return crsd::fail(CRSD_ERR_UNSUPPORTED, "CRSD_PAPER_ELL handle: use crsd_spmv");
    if (!alpha || !beta || !x_padded || !y_local) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    if (((uintptr_t)x_padded | (uintptr_t)y_local) & 15)
        return crsd::fail(CRSD_ERR_INVALID_ARG, "x_padded and y_local must be 16-byte aligned");
    if (c && !A->bound) return crsd::fail(CRSD_ERR_INVALID_ARG, "call crsd_dist_bind first");
    if (c && A->bound_comm != c) return crsd::fail(CRSD_ERR_INVALID_ARG, "handle was bound to another communicator");
    CU_TRY(cudaSetDevice(A->device));
    const size_t es = A->H.elem;
    char *xp = (char *)x_padded;
    const void *xbase = xp + es * A->halo_lo;
    cudaStream_t s = (cudaStream_t)stream;
    int launches = 0;
    crsd_status_t st;
    // The exchange runs on the comm stream (created at the highest stream
    // priority, so its CTAs take the next free SM slots ahead of queued SpMV
    // CTAs). Default order: interior segments launched first, then the
    // exchange — the interior fills the GPU at once and the small exchange
    // kernels slot in as CTAs retire (launching the exchange first measured
    // the same under MPS).
    if (c) CU_TRY(cudaEventRecord(c->ev_x, s));
    // Direct mode (one-sided puts into this handle's crsd_dist_x_alloc
    // buffer) with the JIT kernel: the receive side is fused into the
    // boundary segments' kernel -- each CTA waits for the senders' flags
    // before copying its x windows, the last CTA releases the pads -- so a
    // call is put + interior + boundary, no separate wait / release kernels
    // (CRSD_TUNE_HALO_UNFUSED restores them).
    // Liveness: the boundary CTAs spin until the senders' puts land. A
    // sender on another GPU always runs; a sender SHARING this GPU (ranks
    // co-located, e.g. under MPS) needs an SM slot, which spinning CTAs
    // could all hold -- so with a co-located sender the fused form is used
    // only while the boundary launch fits in one CTA per SM.
    bool colocated_sender = false;
    if (c && c->kind == crsd_comm_s::P2P)
        for (int64_t q : A->recv_peer) colocated_sender |= c->peer_same_gpu[q] != 0;
    const bool fused = c && c->kind == crsd_comm_s::P2P && A->find_dx(xp, c) &&
                       A->variant == VARIANT_JIT && A->jit_halo_function && !A->list_boundary.empty() &&
                       !(A->tune & CRSD_TUNE_HALO_UNFUSED) &&
                       (!colocated_sender || (int64_t)A->list_boundary.size() <= A->sm_count);
    auto exchange = [&]() -> crsd_status_t {
        crsd::NvtxRange nvx("halo exchange");
        CU_TRY(cudaStreamWaitEvent(c->cs, c->ev_x, 0));
        if (c->kind == crsd_comm_s::P2P) {
            ST_TRY(crsd::p2p_exchange(A, c, xp, fused, launches));
        } else {
            const ncclDataType_t ty = (A->H.dtype == CRSD_R64F) ? ncclFloat64 : ncclFloat32;
            NCCL_TRY(ncclGroupStart());
            for (size_t k = 0; k < A->recv_peer.size(); ++k)
                NCCL_TRY(ncclRecv(xp + es * A->recv_off[k], A->recv_count[k], ty, (int)A->recv_peer[k], c->comm,
                                  c->cs));
            for (size_t k = 0; k < A->send_peer.size(); ++k)
                NCCL_TRY(ncclSend(xp + es * A->send_off[k], A->send_count[k], ty, (int)A->send_peer[k], c->comm,
                                  c->cs));
            NCCL_TRY(ncclGroupEnd());
        }
        CU_TRY(cudaEventRecord(c->ev_halo, c->cs));
        return CRSD_OK;
    };
    // a contiguous interior (no scatter column reaching outside: C2, C4, C5)
    // launches as a segment range: no per-CTA list load before the
    // descriptor, and the JIT occupancy classes apply
    const std::vector<int32_t> &li = A->list_interior;
    const bool contig = !li.empty() && (int64_t)li.back() - li.front() + 1 == (int64_t)li.size();
    if (contig)
        st = crsd::run_lists(A, alpha, xbase, beta, y_local, nullptr, li.front(), (int64_t)li.size(), stream,
                             launches);
    else
        st = crsd::run_lists(A, alpha, xbase, beta, y_local, (const int32_t *)A->d_list_interior, 0,
                             (int64_t)li.size(), stream, launches);
    if (st) return st;
    if (c) ST_TRY(exchange());
    // The boundary segments run on the comm stream right behind the
    // exchange, i.e. concurrently with the interior rather than after it: no
    // serial tail (interior drain + a small dependent launch) per call. The
    // caller's stream then waits for the comm stream. CRSD_TUNE_DIST_BOUNDARY_SERIAL
    // runs them on the caller's stream after the interior instead.
    const bool serial = boundary < 0 ? (A->tune & CRSD_TUNE_DIST_BOUNDARY_SERIAL) != 0 : boundary == 1;
    if (c && serial) CU_TRY(cudaStreamWaitEvent(s, c->ev_halo, 0));
    crsd::HaloSync hs;
    if (fused) crsd::make_halo_sync(A, c, hs);
    st = crsd::run_lists(A, alpha, xbase, beta, y_local, (const int32_t *)A->d_list_boundary, 0,
                         (int64_t)A->list_boundary.size(), (c && !serial) ? (void *)c->cs : stream, launches,
                         fused ? &hs : nullptr);
    if (st) return st;
    if (c && c->kind == crsd_comm_s::P2P && !fused) {
        // the pads are free once the boundary segments are done with them
        if (serial) {
            CU_TRY(cudaEventRecord(c->ev_x, s));
            CU_TRY(cudaStreamWaitEvent(c->cs, c->ev_x, 0));
        }
        ST_TRY(crsd::release_halo(A, c));
        ++launches;
    }
    if (c) {
        CU_TRY(cudaEventRecord(c->ev_halo, c->cs));
        CU_TRY(cudaStreamWaitEvent(s, c->ev_halo, 0));
    }
    A->last_launches = launches;
    return st;
}
