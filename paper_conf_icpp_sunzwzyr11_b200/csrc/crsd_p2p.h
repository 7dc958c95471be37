// Peer-memory transport (p2p.cu): symmetric flag block and launch records.
#pragma once

#include <cstdint>

namespace crsd {

constexpr int P2P_MAX_WORLD = 64;
constexpr int P2P_MAX_ITEMS = 16;  // slices per rank and direction (2 per peer; multi-hop)
constexpr int P2P_MAX_RED = 4;     // doubles per scalar allreduce
constexpr int64_t P2P_FLAGS_BYTES = 65536;

// Head of every rank's symmetric region. Slots indexed by the WRITING rank.
struct P2PFlags {
    uint64_t ready[P2P_MAX_WORLD];      // written by sender q: its mailbox holds epoch ready[q]
    uint64_t consumed[P2P_MAX_WORLD];   // written by receiver q: it has read my epoch consumed[q]
    uint64_t red_ready[P2P_MAX_WORLD];  // written by q: red[.][q] holds its epoch red_ready[q]
    double red[2][P2P_MAX_WORLD][P2P_MAX_RED];
    uint64_t halo_epoch;  // own: last completed halo exchange
    uint64_t red_epoch;   // own: last completed allreduce
    uint32_t counter[2];  // own: grid arrival counters (send, recv)
    uint32_t err;         // own: 0, or 1/2/3/4 = send/recv/allreduce/close wait timed out
    int64_t cap;          // own mailbox bytes per parity (read by peers at open)
    uint8_t dev_uuid[16]; // own GPU's UUID (read by peers at open: who shares my GPU)
    uint64_t closing[P2P_MAX_WORLD];  // written by q at crsd_comm_destroy: q no longer touches my region
    // crsd_dist_x_alloc handshake, written by q (host copies into peer memory):
    // q's padded-x IPC handle, then xseq[q] = the allocation's sequence number
    uint8_t xh[P2P_MAX_WORLD][64];
    int64_t xrange[P2P_MAX_WORLD][4];  // {row_begin, row_end, purpose, 0} of the handle q allocated it for
    uint64_t xseq[P2P_MAX_WORLD];
};
static_assert(sizeof(P2PFlags) <= P2P_FLAGS_BYTES, "P2PFlags too large");

struct P2PItem {
    const void *src;
    void *dst;
    int64_t bytes;
    int64_t parity_shift;  // bytes from mailbox parity 0 to parity 1 of the mailbox this item touches
};

struct P2PLaunch {
    P2PFlags *local;
    P2PFlags *peer_flags[P2P_MAX_ITEMS];  // per distinct peer of this direction
    int32_t peer[P2P_MAX_ITEMS];
    int32_t npeer, nitems, rank, pad_;
    uint64_t timeout_ns;
    P2PItem items[P2P_MAX_ITEMS];
};

struct P2PReduce {
    P2PFlags *local;
    P2PFlags *peer_flags[P2P_MAX_WORLD];
    int32_t rank, world;
    uint64_t timeout_ns;
};

int p2p_launch_send(const P2PLaunch &L, int grid, void *stream);
int p2p_launch_recv(const P2PLaunch &L, int grid, void *stream);
int p2p_launch_put(const P2PLaunch &L, int grid, void *stream);
int p2p_launch_wait(const P2PLaunch &L, void *stream);
int p2p_launch_release(const P2PLaunch &L, void *stream);
int p2p_launch_allreduce(const P2PReduce &R, double *val, int n, void *stream);
int p2p_launch_close(const P2PReduce &R, uint64_t token, void *stream);

}  // namespace crsd
