// Opaque handle types behind crsd_matrix_t / crsd_comm_t.
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "crsd_internal.h"

struct crsd_matrix_s {
    crsd::HostCRSD H;
    bool host_only = false;
    bool host_vals_dropped = false;
    int device = -1;
    int sm_count = 148;
    int rpt = 2;
    int variant = crsd::VARIANT_LDG;
    int64_t smem_bytes = 0;
    int64_t xmax_elems = 0;
    int tma_split = 1, tma_q = 2;
    // JIT variant: generated source, loaded module and kernel (CUmodule / CUfunction)
    std::string jit_source;
    void *jit_module = nullptr;
    void *jit_function = nullptr;
    void *jit_halo_function = nullptr;  // the same codelets with the fused halo receive (crsd_jit_halo)
    void *jit_rs_function = nullptr;    // register-staged codelets (crsd_jit_rs)
    int regstage = -1;                  // register staging in use (jit_decide; -1: not decided yet)
    std::vector<char> jit_cubin;    // the compiled codelets (crsd_jit_cubin)
    int32_t jit_chunk = 0;          // opts.jit_chunk: diagonals per staging chunk (0 = per x window, <0 = one)
    uint32_t tune = 0;              // opts.tune: CRSD_TUNE_* switches
    int32_t e2e_chunks = 0;         // opts.e2e_chunks: crsd_spmv_host pipeline depth (0: from the size)
    // one-GPU launches of the one-shot codelets split into contiguous segment
    // ranges of equal occupancy class: {seg_begin, seg_count, dynamic smem}
    // {seg_begin, seg_count, dynamic smem, aux}: aux = 1 for short runs that
    // go to a forked stream alongside the main sequence
    std::vector<std::vector<int64_t>> jit_ranges;
    std::vector<void *> jit_pool;       // cudaStream_t: forked streams for range launches
    std::vector<void *> jit_ev_join;    // cudaEvent_t, one per pool stream
    void *jit_ev_fork = nullptr;        // cudaEvent_t
    int64_t tma_smem = 0;
    std::vector<int32_t> plan;
    int32_t last_launches = 0;
    int64_t device_bytes = 0;

    // x layout (relative to the local x base)
    int64_t halo_lo = 0, halo_hi = 0;              // allocated pads (halo_lo multiple of 4)
    int64_t halo_lo_valid = 0, halo_hi_valid = 0;  // elements actually exchanged
    int64_t x_lo = 0, x_hi = 0;                    // valid x range

    std::vector<crsd::SegDesc> segdesc;
    std::vector<int32_t> list_interior, list_boundary;
    int64_t nedge = 0;

    // device arrays
    void *d_vals = nullptr;
    void *d_segs = nullptr;
    void *d_offs = nullptr;
    void *d_plan = nullptr;
    void *d_scat_row = nullptr;
    void *d_scat_col = nullptr;
    void *d_scat_val = nullptr;
    void *d_scat_rec = nullptr;
    void *d_scat_slab = nullptr;  // crsd::SlabRec[nseg * SLAB_K] (JIT; null if a column does not fit int32)
    void *d_list_interior = nullptr;
    void *d_list_boundary = nullptr;
    void *d_list_all_edge = nullptr;
    void *d_ell_rowno = nullptr;  // CRSD_PAPER_ELL: scatter rows stored whole (int64 local rows)
    void *d_ell_col = nullptr;    // int64, column-major, -1 padded
    void *d_ell_val = nullptr;
    void *d_x_scratch = nullptr;
    void *d_y_scratch = nullptr;

    // end-to-end pipeline (crsd_spmv_host): row chunks, x chunks, streams
    bool e2e_ready = false;
    int e2e_nchunk = 0;
    std::vector<int64_t> e2e_seg;      // nchunk + 1 segment boundaries
    std::vector<int64_t> e2e_xcut;     // nchunk + 1 x element boundaries
    std::vector<int> e2e_need;         // last x chunk each row chunk needs
    void *e2e_h2d = nullptr, *e2e_d2h = nullptr;  // cudaStream_t
    std::vector<void *> e2e_ev_x, e2e_ev_y;         // cudaEvent_t
    void *e2e_ev_start = nullptr, *e2e_ev_done = nullptr;

    // CG workspace (crsd_cg): state, partials, history, r, q, halo-padded p
    void *d_cg = nullptr;
    int64_t cg_bytes = 0;
    void *cg_stream = nullptr;                  // cudaStream_t (graph capture / replay)
    void *cg_ev_in = nullptr, *cg_ev_out = nullptr;  // cudaEvent_t

    // multi-GPU plan (crsd_dist_bind)
    bool bound = false;
    std::vector<int64_t> recv_peer, recv_off, recv_count;  // offsets into x_padded
    std::vector<int64_t> send_peer, send_off, send_count;
    // peer-memory transport: byte offsets into my mailbox (sends) / the sender's mailbox (recvs)
    std::vector<int64_t> send_mb_off, recv_mb_off;
    const void *bound_comm = nullptr;
    std::vector<int64_t> range_table;  // every rank's {row_begin, row_end, halo_lo_valid, halo_hi_valid}
    // direct (one-sided put) mode: padded x buffers allocated by the library
    // (IPC-exported) with every peer's counterpart mapped; the sends land in
    // the peers' pads. purpose 0: crsd_dist_x_alloc (the caller's x), 1: the
    // CG's p (so a CG never writes into the caller's x)
    struct DirectX {
        void *own = nullptr;
        std::vector<void *> peer;
        const void *comm = nullptr;
        int purpose = 0;
    };
    std::vector<DirectX> dx;
    const DirectX *find_dx(const void *xp, const void *comm) const {
        for (const DirectX &d : dx)
            if (d.own == xp && d.comm == comm) return &d;
        return nullptr;
    }
};

namespace crsd {
void free_device(crsd_matrix_s *A);
std::string jit_generate(const crsd_matrix_s *A);
crsd_status_t jit_build(crsd_matrix_s *A);
void jit_free(crsd_matrix_s *A);
template <typename T>
int jit_launch(const crsd_matrix_s *A, const SpmvArgs<T> &a, void *stream);
// crsd_spmv launches A's JIT kernel with programmatic dependent launch
bool jit_pdl(const crsd_matrix_s *A);
// A's scatter points go to the per-segment slab (SlabRec) for the JIT codelets
bool slab_ok(const crsd_matrix_s *A);
// Run the SpMV kernel over a device list of segments (list == nullptr: the
// segment range [seg_begin, seg_begin + count)). x_base is the local x base
// (x_padded + halo_lo).
// halo != null: the boundary launch of a direct-mode exchange with the
// receive side fused into the JIT kernel (crsd_jit_halo).
// pdl: the caller (crsd_spmv) allows a programmatic dependent launch
// (used when jit_pdl(A) and the stream is not capturing).
crsd_status_t run_lists(crsd_matrix_s *A, const void *alpha, const void *x_base, const void *beta, void *y,
                        const int32_t *list, int64_t seg_begin, int64_t count, void *stream, int &launches,
                        const HaloSync *halo = nullptr, bool pdl = false);
}  // namespace crsd
