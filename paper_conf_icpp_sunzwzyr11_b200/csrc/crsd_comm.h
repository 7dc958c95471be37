// Communicator behind crsd_comm_t (dist.cpp, solver.cpp): NCCL, or the
// library's own peer-memory transport (p2p.cu) over CUDA-IPC-mapped regions.
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>

#include <vector>

#include "crsd.h"
#include "crsd_p2p.h"

struct crsd_matrix_s;

struct crsd_comm_s {
    enum Kind { NCCL = 0, P2P = 1 };
    int kind = NCCL;
    ncclComm_t comm = nullptr;
    int rank = 0, world = 1, device = 0;
    cudaStream_t cs = nullptr;                         // halo exchange stream
    cudaEvent_t ev_x = nullptr, ev_halo = nullptr;
    // P2P: own symmetric region [P2PFlags | mailbox parity 0 | parity 1] and the peers' (IPC-opened)
    void *sym = nullptr;
    int64_t cap = 0;                  // bytes per mailbox parity
    std::vector<void *> peer_sym;     // world entries, nullptr for self / not opened
    std::vector<int64_t> peer_cap;    // each peer's mailbox bytes per parity (read from its flags)
    std::vector<uint8_t> peer_same_gpu;  // 1 if the peer's region lives on my GPU (ranks sharing a device)
    bool opened = false;
    bool poisoned = false;            // a wait timed out (seen by crsd_comm_error): refuse further exchanges
    uint64_t xseq = 0;                // crsd_dist_x_alloc handshakes made
    uint64_t timeout_ns = 30ull * 1000 * 1000 * 1000;  // peer-memory waits (CRSD_P2P_TIMEOUT_S)
};

namespace crsd {
// Sum n doubles (device pointer) over every rank of comm, in place, on stream.
crsd_status_t comm_allreduce_f64(crsd_comm_s *c, double *dev, int n, cudaStream_t stream);
// crsd_spmv_dist with the boundary placement chosen by the caller: -1 default,
// 0 concurrent with the interior (comm stream), 1 serial after the interior
// the handle's crsd_dist_x_alloc buffer (direct one-sided puts), collective
crsd_status_t dist_x_alloc(crsd_matrix_s *A, crsd_comm_s *c, int purpose, void **out);
crsd_status_t release_halo(crsd_matrix_s *A, crsd_comm_s *c);
crsd_status_t spmv_dist_impl(crsd_matrix_s *A, const void *alpha, void *x_padded, const void *beta, void *y_local,
                             crsd_comm_s *c, void *stream, int boundary);
}  // namespace crsd
