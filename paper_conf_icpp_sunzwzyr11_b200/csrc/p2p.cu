// Peer-memory transport for the row-partitioned SpMV (BASELINE.json
// north_star (3)): the x halo exchange and the
// CG's scalar allreduce done by our own kernels through CUDA-IPC-mapped
// device memory (NVLink / NVSwitch loads and stores between GPUs; plain HBM
// when two ranks share one GPU), instead of NCCL calls.
//
// Each rank owns one symmetric region (cudaMalloc, exported with
// cudaIpcGetMemHandle, opened by every peer):
//
//   [P2PFlags (64 KB slot)] [mailbox parity 0 (cap bytes)] [mailbox parity 1 (cap bytes)]
//
// Two ways to move the halo of call e (the epoch, device-resident, so the
// kernels can be captured into a CUDA graph):
//
// Direct (one-sided put; x_padded allocated by crsd_dist_x_alloc, so every
// rank has every neighbour's padded x mapped):
//   p2p_put:     wait until each receiver has released epoch e-1 (its
//                boundary segments of call e-1 no longer read its pads:
//                my flags.consumed[q] >= e-1); store my send slices straight
//                into the receivers' pads over NVLink; last CTA: system
//                fence, flags.ready[me] = e in each receiver's region.
//   p2p_wait:    wait until every sender has published e (flags.ready[q] >= e).
//   (boundary segments run here, reading the pads)
//   p2p_release: flags.consumed[me] = e in each sender's region, my halo
//                epoch = e.
// One NVLink crossing per halo byte; no mailbox copy.
//
// Mailbox (two-stage; any caller-owned x_padded):
//   p2p_send:    wait until every peer I send to has released epoch e-2;
//                copy my send slices into mailbox[e&1]; last CTA: system
//                fence, flags.ready[me] = e in each receiver's region.
//   p2p_recv:    wait for flags.ready[q] >= e; pull the slices from the
//                peers' mailbox[e&1] into the pads of x_padded.
//   (boundary segments)  p2p_release as above.
// Two parities let a sender run one call ahead of a slow receiver.
//
// Scalar allreduce (CG dots, n <= 4 doubles): one thread writes its values
// into every peer's red[e&1][me] slot, fences, publishes red_ready[me] = e,
// waits for red_ready[q] >= e from every peer and sums the W slots in rank
// order 0..W-1 — the same operands in the same order on every rank, so every
// rank gets the bit-identical result (deterministic, unlike a ring).
//
// Every wait is bounded (%globaltimer; 30 s unless CRSD_P2P_TIMEOUT_S says
// otherwise): on timeout the kernel sets flags.err. A communicator with err
// set is poisoned: every later kernel skips its copies and publishes
// nothing (but still keeps its grid counters and epochs consistent), and
// crsd_comm_error reports the code; the results are then invalid.
#include <cuda_runtime.h>

#include <cstdint>

#include "crsd_p2p.h"

namespace crsd {

namespace {

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t *p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ bool poisoned(P2PFlags *me) { return *(volatile uint32_t *)&me->err != 0; }

// Spin until *p >= want (acquire, system scope). Returns false after
// timeout_ns (crsd_comm_s::timeout_ns, CRSD_P2P_TIMEOUT_S, default 30 s).
__device__ bool wait_geq(const uint64_t *p, uint64_t want, uint64_t timeout_ns) {
    if (ld_acquire_sys(p) >= want) return true;
    const uint64_t t0 = globaltimer();
    while (ld_acquire_sys(p) < want) {
        __nanosleep(200);
        if (globaltimer() - t0 > timeout_ns) return false;
    }
    return true;
}

// Byte copy of the items, split over the grid in 4-byte words (element
// sizes are 4 or 8; slices start at arbitrary elements, so 16-B alignment is
// not guaranteed and the halo is ~2 % of a rank's bytes). Parity 1 of a
// mailbox lies parity_shift bytes after parity 0: added to the destination
// (send: my mailbox) or to the source (recv: the sender's mailbox); direct
// puts have parity_shift 0.
__device__ void copy_items(const P2PItem *items, int nitems, bool odd, bool shift_dst, int64_t gtid, int64_t gsz) {
    for (int k = 0; k < nitems; ++k) {
        const int64_t sh = odd ? items[k].parity_shift : 0;
        const uint32_t *s = (const uint32_t *)((const char *)items[k].src + (shift_dst ? 0 : sh));
        uint32_t *d = (uint32_t *)((char *)items[k].dst + (shift_dst ? sh : 0));
        const int64_t nw = items[k].bytes >> 2;
        if ((((uintptr_t)s | (uintptr_t)d) & 15) == 0) {
            const int64_t nv = nw >> 2;
            const uint4 *s4 = (const uint4 *)s;
            uint4 *d4 = (uint4 *)d;
            for (int64_t i = gtid; i < nv; i += gsz) d4[i] = __ldcv(s4 + i);
            for (int64_t i = (nv << 2) + gtid; i < nw; i += gsz) d[i] = __ldcv(s + i);
        } else {
            for (int64_t i = gtid; i < nw; i += gsz) d[i] = __ldcv(s + i);
        }
    }
}

// Grid arrival: returns true in exactly one CTA (the last to arrive), after
// every CTA's writes are fenced at system scope. Every CTA must call it,
// also after a failed wait, so the counter returns to 0 for the next launch.
__device__ bool last_cta(uint32_t *counter) {
    __shared__ bool last;
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) {
        const uint32_t prev = atomicAdd(counter, 1u);
        last = (prev == gridDim.x - 1);
        if (last) *counter = 0;  // reset for the next launch (stream-ordered)
    }
    __syncthreads();
    if (last) __threadfence_system();
    return last;
}

// Thread 0 of every CTA: is the communicator healthy and has every listed
// peer reached `want` in flags slot `slot` (ready or consumed)? On timeout
// sets err = code.
__device__ int ready_to_go(P2PLaunch &L, const uint64_t *slot, uint64_t want, uint32_t code) {
    __shared__ int ok;
    if (threadIdx.x == 0) {
        ok = !poisoned(L.local);
        for (int k = 0; ok && k < L.npeer; ++k)
            if (!wait_geq(&slot[L.peer[k]], want, L.timeout_ns)) {
                ok = 0;
                atomicExch(&L.local->err, code);
            }
    }
    __syncthreads();
    return ok;
}

// mailbox mode, sender side
__global__ void p2p_send_kernel(P2PLaunch L) {
    P2PFlags *me = L.local;
    const uint64_t e = *(volatile uint64_t *)&me->halo_epoch + 1;
    const int ok = ready_to_go(L, me->consumed, e > 2 ? e - 2 : 0, 1);
    const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t gsz = (int64_t)gridDim.x * blockDim.x;
    // items carry parity-0 mailbox destinations (my mailbox, my capacity)
    if (ok) copy_items(L.items, L.nitems, (e & 1) != 0, true, gtid, gsz);
    if (last_cta(&me->counter[0]) && threadIdx.x == 0 && !poisoned(me))
        for (int k = 0; k < L.npeer; ++k) st_release_sys(&L.peer_flags[k]->ready[L.rank], e);
}

// mailbox mode, receiver side
__global__ void p2p_recv_kernel(P2PLaunch L) {
    P2PFlags *me = L.local;
    const uint64_t e = *(volatile uint64_t *)&me->halo_epoch + 1;
    const int ok = ready_to_go(L, me->ready, e, 2);
    const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t gsz = (int64_t)gridDim.x * blockDim.x;
    // items carry parity-0 sources in the SENDER's mailbox, shifted by the
    // sender's capacity for parity 1 (capacities may differ per rank)
    if (ok) copy_items(L.items, L.nitems, (e & 1) != 0, false, gtid, gsz);
    last_cta(&me->counter[1]);
}

// direct mode: one-sided put into the receivers' pads
__global__ void p2p_put_kernel(P2PLaunch L) {
    P2PFlags *me = L.local;
    const uint64_t e = *(volatile uint64_t *)&me->halo_epoch + 1;
    const int ok = ready_to_go(L, me->consumed, e - 1, 1);
    const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t gsz = (int64_t)gridDim.x * blockDim.x;
    if (ok) copy_items(L.items, L.nitems, false, true, gtid, gsz);
    if (last_cta(&me->counter[0]) && threadIdx.x == 0 && !poisoned(me))
        for (int k = 0; k < L.npeer; ++k) st_release_sys(&L.peer_flags[k]->ready[L.rank], e);
}

// direct mode: every sender's slices have landed in my pads
__global__ void p2p_wait_kernel(P2PLaunch L) {
    P2PFlags *me = L.local;
    const uint64_t e = *(volatile uint64_t *)&me->halo_epoch + 1;
    ready_to_go(L, me->ready, e, 2);
}

// both modes, after the boundary segments: my pads of epoch e are free
__global__ void p2p_release_kernel(P2PLaunch L) {
    if (threadIdx.x != 0) return;
    P2PFlags *me = L.local;
    const uint64_t e = *(volatile uint64_t *)&me->halo_epoch + 1;
    if (!poisoned(me))
        for (int k = 0; k < L.npeer; ++k) st_release_sys(&L.peer_flags[k]->consumed[L.rank], e);
    me->halo_epoch = e;
}

__global__ void p2p_allreduce_kernel(P2PReduce R, double *val, int n) {
    if (threadIdx.x != 0) return;
    P2PFlags *me = R.local;
    const uint64_t e = me->red_epoch + 1;
    me->red_epoch = e;
    if (poisoned(me)) return;
    const int par = (int)(e & 1);
    double v[P2P_MAX_RED];
    for (int i = 0; i < n; ++i) v[i] = val[i];
    for (int q = 0; q < R.world; ++q) {
        if (q == R.rank) continue;
        P2PFlags *pf = R.peer_flags[q];
        for (int i = 0; i < n; ++i) *(volatile double *)&pf->red[par][R.rank][i] = v[i];
    }
    __threadfence_system();
    for (int q = 0; q < R.world; ++q)
        if (q != R.rank) st_release_sys(&R.peer_flags[q]->red_ready[R.rank], e);
    bool ok = true;
    for (int q = 0; q < R.world; ++q)
        if (q != R.rank && !wait_geq(&me->red_ready[q], e, R.timeout_ns)) ok = false;
    if (!ok) {
        atomicExch(&me->err, 3u);
        return;
    }
    double s[P2P_MAX_RED];
    for (int i = 0; i < n; ++i) s[i] = 0.0;
    for (int q = 0; q < R.world; ++q)
        for (int i = 0; i < n; ++i) s[i] += (q == R.rank) ? v[i] : *(volatile double *)&me->red[par][q][i];
    for (int i = 0; i < n; ++i) val[i] = s[i];
}

// Collective close: tell every peer I am done with its region and wait
// (bounded) until every peer says the same about mine; only then may the
// host unmap the peers' regions and free its own.
__global__ void p2p_close_kernel(P2PReduce R, uint64_t token) {
    if (threadIdx.x != 0) return;
    P2PFlags *me = R.local;
    for (int q = 0; q < R.world; ++q)
        if (q != R.rank) st_release_sys(&R.peer_flags[q]->closing[R.rank], token);
    for (int q = 0; q < R.world; ++q)
        if (q != R.rank && !wait_geq(&me->closing[q], token, R.timeout_ns)) atomicExch(&me->err, 4u);
}

}  // namespace

int p2p_launch_send(const P2PLaunch &L, int grid, void *stream) {
    p2p_send_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>(L);
    return (int)cudaGetLastError();
}
int p2p_launch_recv(const P2PLaunch &L, int grid, void *stream) {
    p2p_recv_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>(L);
    return (int)cudaGetLastError();
}
int p2p_launch_put(const P2PLaunch &L, int grid, void *stream) {
    p2p_put_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>(L);
    return (int)cudaGetLastError();
}
int p2p_launch_wait(const P2PLaunch &L, void *stream) {
    p2p_wait_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(L);
    return (int)cudaGetLastError();
}
int p2p_launch_release(const P2PLaunch &L, void *stream) {
    p2p_release_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(L);
    return (int)cudaGetLastError();
}
int p2p_launch_allreduce(const P2PReduce &R, double *val, int n, void *stream) {
    p2p_allreduce_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(R, val, n);
    return (int)cudaGetLastError();
}
int p2p_launch_close(const P2PReduce &R, uint64_t token, void *stream) {
    p2p_close_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(R, token);
    return (int)cudaGetLastError();
}

}  // namespace crsd
