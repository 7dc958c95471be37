/*
 * crsd.h -- C-ABI of the B200-native CRSD SpMV library (libcrsd.so).
 *
 * Operation (PAPER.md P:L33-39 problem statement; "the result
 * should be stored at ... destination vector y"; generalised to BLAS form by
 * BASELINE.json north_star (1)):
 *
 *     y = alpha * A * x + beta * y
 *
 * for a diagonal sparse matrix A stored in CRSD, "Compressed Row Segment with
 * Diagonal-pattern" (§II; Fig. 4):
 *   - rows are split into row segments of `mrows` rows;
 *   - in each segment the diagonals (offset = col - row) that
 *     carry >= 2 nonzeros, or that belong to a run bridged across idle
 *     sections of <= idle_max zeros, are stored (R1/R2);
 *   - consecutive segments with the same diagonal set form a diagonal
 *     pattern, grouped into AD / NAD groups;
 *   - values are stored contiguously per segment and per diagonal, filled
 *     zeros included (address formula P:L613-623);
 *   - the remaining nonzeros are scatter points, stored separately
 *     (per-segment list, R5).
 * At SpMV time only values are read; no per-nonzero index is loaded
 * (P:L631-635).
 *
 * Conventions for every call
 *   - Every call returns crsd_status_t; CRSD_OK == 0. No call throws, aborts
 *     or exits. crsd_last_error() returns a thread-local message describing
 *     the last non-OK status of the calling thread.
 *   - Pointers documented as HOST must be host-accessible; DEVICE pointers
 *     must be device memory of the handle's CUDA device. Ownership is stated
 *     per argument; the library never frees caller memory.
 *   - `stream` arguments are cudaStream_t values passed as void* (NULL = the
 *     legacy default stream). Device calls are asynchronous and
 *     stream-ordered unless stated; launch errors are returned synchronously,
 *     asynchronous kernel faults surface at the caller's next synchronisation.
 *   - A handle must not be used by two threads at once.
 *   - The library holds no global state besides the thread-local error text.
 */
#ifndef CRSD_H
#define CRSD_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    CRSD_OK = 0,
    CRSD_ERR_INVALID_ARG = 1, /* NULL where not allowed, bad size, misaligned device pointer, ... */
    CRSD_ERR_INDEX_RANGE = 2, /* a COO row/col outside [0,nrows)x[0,ncols) (or outside the handle's row range) */
    CRSD_ERR_DUPLICATE = 3,   /* a (row,col) given twice and CRSD_SUM_DUPLICATES not set */
    CRSD_ERR_UNSUPPORTED = 4, /* valid request the GPU path does not handle (e.g. mrows not a multiple of 32*RPT) */
    CRSD_ERR_ALLOC = 5,       /* host or device allocation failed */
    CRSD_ERR_CUDA = 6,        /* a CUDA runtime call or kernel launch failed */
    CRSD_ERR_NCCL = 7         /* an NCCL call failed */
} crsd_status_t;

typedef enum { CRSD_R32F = 0, CRSD_R64F = 1 } crsd_dtype_t;

/* opts.flags */
#define CRSD_SUM_DUPLICATES 0x1u /* duplicates are summed (in input order) instead of rejected */
#define CRSD_HOST_ONLY 0x2u      /* build the CRSD structure on the host only (export/inspection); no device memory is touched and crsd_spmv* return CRSD_ERR_UNSUPPORTED */
#define CRSD_DROP_ZEROS 0x4u     /* explicit zero entries are dropped instead of kept in the scatter list (R10) */
#define CRSD_PAPER_ELL 0x8u      /* paper-exact scatter handling: every row holding a
                                    scatter point is also stored whole in ELL and, after the diagonal part, its
                                    y is OVERWRITTEN by the ELL row product, accumulated in ascending column
                                    order with separately rounded multiplies and adds (CSR order). crsd_spmv
                                    then needs beta == 0 (the paper computes y = A x; UNSUPPORTED otherwise);
                                    one-GPU handles only; crsd_spmv_host / _dist / crsd_cg return UNSUPPORTED.
                                    DESIGN.md R5/R6, §8(f) NEXT 3. */

/*
 * Build options. Call crsd_opts_init() for defaults (NULL opts == defaults).
 *   mrows     row-segment height (token `mrows`); 0 => 2 KB of
 *             values per diagonal run: 256 (fp64) / 512 (fp32), except that
 *             fp32 falls back to 256 when a segment's staging at 512 rows
 *             would leave fewer than 4 CTAs per SM. The
 *             GPU path needs mrows % (32*RPT) == 0 and mrows <= 256*RPT,
 *             RPT = 2 rows per thread for fp64 and 4 for fp32 (one 128-bit
 *             vector per thread and diagonal; <= 256 threads per CTA); the
 *             host builder accepts any mrows >= 1.
 *   idle_max  longest run of zeros along a diagonal that is bridged by
 *             filling zeros (R2); < 0 => mrows - 1.
 *   flags     CRSD_* flags above.
 *   row_begin, row_end
 *             rows owned by this handle for the row-partitioned multi-GPU
 *             path; both 0 => all rows [0, nrows). COO rows must lie in the
 *             range. row_begin must be a multiple of mrows.
 *   device    CUDA device ordinal the handle's memory lives on (-1 => current).
 *   nthreads  host builder threads (OpenMP); 0 => OpenMP default.
 *   variant   GPU kernel: CRSD_VARIANT_AUTO (0), CRSD_VARIANT_LDG (1: 128-bit
 *             register loads, x by warp shuffle), CRSD_VARIANT_TMA (2: one CTA
 *             per segment, bulk copies of its values and x windows into
 *             shared memory) or CRSD_VARIANT_PIPE (3: persistent CTAs, a
 *             producer warp streams value chunks through a shared-memory
 *             ring with TMA bulk copies) or CRSD_VARIANT_JIT (4: the TMA
 *             data movement with every pattern quantity baked into a
 *             runtime-generated codelet, NVRTC; the paper's code generator,
 *             P:L131-143). AUTO picks JIT when a segment stages in <= 75 KB
 *             (TMA for <= 32 KB unsplit segments if NVRTC is unavailable),
 *             PIPE for larger ones, LDG when neither staging fits in shared
 *             memory. DESIGN.md "Kernels".
 */
typedef struct {
    int32_t mrows;
    int32_t idle_max;
    uint32_t flags;
    int32_t device;
    int64_t row_begin;
    int64_t row_end;
    int32_t nthreads;
    int32_t variant;
    int32_t jit_chunk;  /* JIT staging chunks (each its own mbarrier): 0 => one per x
                           window (default), k > 0 => windows split into runs of <= k diagonals, < 0 =>
                           the whole segment on one mbarrier */
    uint32_t tune;      /* CRSD_TUNE_* implementation switches (0 = the measured defaults); per handle */
    int32_t e2e_chunks; /* crsd_spmv_host pipeline depth (row chunks); 0 => x bytes / 56 MB, within [16, 64] */
    int32_t reserved;   /* must be 0 */
} crsd_opts_t;

/* opts.tune: the alternatives the measurements in DESIGN.md compare against
 * the defaults. They change how the work is scheduled, never what is
 * computed (every setting gives the same y bit for bit). */
#define CRSD_TUNE_JIT_DESC_ISSUE 0x1u      /* JIT: issue the bulk copies after loading the segment descriptor
                                              instead of from the baked instance lookup */
#define CRSD_TUNE_JIT_ONE_LAUNCH 0x2u      /* JIT: one launch for the whole matrix (no occupancy-class ranges) */
#define CRSD_TUNE_JIT_SPLIT_ALL 0x4u       /* JIT: a range launch at every occupancy-class change (testing) */
#define CRSD_TUNE_JIT_SEQUENTIAL 0x8u      /* JIT: range launches one after another instead of concurrently */
#define CRSD_TUNE_DIST_BOUNDARY_SERIAL 0x10u /* crsd_spmv_dist / crsd_cg: boundary segments after the interior on
                                              the caller's stream instead of behind the exchange on the comm stream */
#define CRSD_TUNE_NO_JIT 0x20u             /* AUTO never picks the JIT variant */
#define CRSD_TUNE_HALO_UNFUSED 0x40u       /* crsd_spmv_dist direct mode: separate wait / release kernels instead of
                                              the receive fused into the boundary kernel (crsd_jit_halo) */
#define CRSD_TUNE_JIT_NO_SLAB 0x100u       /* JIT: each CTA finds its scatter points through its segment descriptor
                                              instead of the per-segment slab of the first 16 */
#define CRSD_TUNE_JIT_NO_REGSTAGE 0x200u   /* JIT, one GPU: no register staging. By default, when staging the last
                                              diagonals of the heavy patterns in registers (one more CTA per SM)
                                              lets the handle run as one launch instead of occupancy-class
                                              ranges, those segments run in a second kernel; DESIGN.md "Kernels" */
#define CRSD_TUNE_JIT_NO_PDL 0x80u         /* crsd_spmv, JIT: plain launches instead of programmatic dependent launch.
                                              By default a one-GPU handle whose matrix runs as ONE launch is
                                              launched with PDL: it may start while the previous kernel on the
                                              stream drains; its CTAs stream the (immutable) matrix values first
                                              and wait for the previous kernel (griddepcontrol.wait) before they
                                              touch x or y. Handles split into occupancy-class ranges keep their
                                              concurrent range launches; stream capture keeps plain launches */

#define CRSD_VARIANT_AUTO 0
#define CRSD_VARIANT_LDG 1
#define CRSD_VARIANT_TMA 2
#define CRSD_VARIANT_PIPE 3
#define CRSD_VARIANT_JIT 4

typedef struct crsd_matrix_s *crsd_matrix_t;
typedef struct crsd_comm_s *crsd_comm_t;

/* Sizes and counts of a built matrix (all counts are of the local rows for a
 * row-partitioned handle). */
typedef struct {
    int64_t nrows, ncols;           /* global dimensions */
    int64_t row_begin, row_end;     /* owned rows */
    int32_t mrows, idle_max;
    int32_t dtype;                  /* crsd_dtype_t */
    int32_t rows_per_thread;        /* RPT of the GPU kernel (2 fp64, 4 fp32) */
    int64_t nnz;                    /* canonical entries (after duplicate handling) */
    int64_t nseg;                   /* row segments */
    int64_t ninst;                  /* pattern instances = the paper's diagonal patterns (Table II rows) */
    int64_t npat;                   /* distinct diagonal-offset sets */
    int64_t noffsets;               /* sum over distinct patterns of NDias */
    int64_t max_ndias;              /* max NDias over patterns */
    int64_t nslots;                 /* stored diagonal slots = sum NRS_p * NNzRS_p */
    int64_t ndiag_nnz;              /* nonzeros stored on diagonals */
    int64_t nfills;                 /* filled zeros = nslots - ndiag_nnz */
    int64_t nscatter;               /* scatter entries */
    int64_t nedge_seg;              /* segments run by the guarded (edge) kernel body */
    int64_t halo_lo, halo_hi;       /* x halo pads (elements) of a row-partitioned handle; halo_lo is a multiple of 4 */
    int64_t halo_lo_valid, halo_hi_valid; /* halo elements actually exchanged (<= the pads; clipped at the matrix edges) */
    int64_t device_bytes;           /* device memory held by the handle */
    int32_t variant;                /* kernel variant in use (CRSD_VARIANT_LDG / _TMA / _PIPE / _JIT) */
    int32_t smem_bytes;             /* dynamic shared memory per CTA of the TMA variant */
    int64_t unique_bytes_beta0;     /* algorithmic bytes of one SpMV with beta == 0 */
    int64_t unique_bytes_beta1;     /* ... with beta != 0 (y also read) */
    int32_t jit_launches;           /* JIT: kernel launches of one crsd_spmv (occupancy-class ranges), else 1 */
    int32_t pdl;                    /* 1: crsd_spmv launches with programmatic dependent launch (CRSD_TUNE_JIT_NO_PDL) */
    int32_t regstage;               /* 1: register staging in use -- crsd_spmv launches the register-staged kernel
                                       (crsd_jit_rs) for some segments (CRSD_TUNE_JIT_NO_REGSTAGE) */
    int32_t reserved_;
} crsd_info_t;

/*
 * Host copies of the CRSD structure (B200 layout).
 * Sizes come from crsd_info_t; any NULL pointer is skipped. Caller-owned.
 *   inst_first_seg[ninst], inst_nseg[ninst], inst_pattern[ninst]
 *   pat_ptr[npat+1], pat_offsets[noffsets]  (ascending offsets per pattern)
 *   vals[nslots]  (dtype) -- instance i, local segment g, diagonal d, row l at
 *                 base_i + g*NDias*mrows + d*mrows + l, base_i = sum_{j<i}
 *                 nseg_j*NDias_j*mrows
 *   scat_ptr[nseg+1], scat_row[nscatter] (row within segment),
 *   scat_col[nscatter] (global column), scat_val[nscatter] (dtype);
 *   entries of a segment sorted by (row, col).
 */
typedef struct {
    int64_t *inst_first_seg;
    int64_t *inst_nseg;
    int32_t *inst_pattern;
    int64_t *pat_ptr;
    int64_t *pat_offsets;
    void *vals;
    int64_t *scat_ptr;
    int32_t *scat_row;
    int64_t *scat_col;
    void *scat_val;
} crsd_export_t;

const char *crsd_last_error(void);
const char *crsd_version(void);
crsd_status_t crsd_opts_init(crsd_opts_t *opts);

/*
 * Build a CRSD matrix from COO (§II; steps in DESIGN.md "Builder").
 *   nrows, ncols   global dimensions, > 0 and < 2^31.
 *   nnz            entries, >= 0.
 *   row, col       HOST int64[nnz], caller-owned, read-only, copied. Any order.
 *   val            HOST dtype[nnz] (float or double), caller-owned, copied.
 *   dtype          CRSD_R32F or CRSD_R64F.
 *   opts           NULL => defaults.
 *   out            receives the handle (NULL on failure).
 * Errors: INVALID_ARG, INDEX_RANGE, DUPLICATE, UNSUPPORTED, ALLOC, CUDA.
 * Synchronous: the device copy is complete when the call returns.
 */
crsd_status_t crsd_create_from_coo(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row,
                                   const int64_t *col, const void *val, crsd_dtype_t dtype,
                                   const crsd_opts_t *opts, crsd_matrix_t *out);

/* Same from CSR: row_ptr HOST int64[nrows_local+1] over the owned rows
 * (row_ptr[0] may be nonzero: entries are col[row_ptr[0]..row_ptr[n]]). */
crsd_status_t crsd_create_from_csr(int64_t nrows, int64_t ncols, const int64_t *row_ptr, const int64_t *col,
                                   const void *val, crsd_dtype_t dtype, const crsd_opts_t *opts,
                                   crsd_matrix_t *out);

/* Destroy a handle and free its device/host memory. NULL is a no-op. Not
 * stream-ordered: the caller must ensure no SpMV on the handle is in flight. */
crsd_status_t crsd_destroy(crsd_matrix_t A);

/*
 * y = alpha*A*x + beta*y on the GPU (P:L567-719 method; kernels DESIGN.md §Kernels).
 *   alpha, beta    HOST pointers to one scalar of the matrix dtype.
 *   x              DEVICE dtype[ncols], 16-byte aligned, read-only.
 *   y              DEVICE dtype[nrows], 16-byte aligned; not read when
 *                  *beta == 0 (BLAS convention). Must not alias x.
 *   stream         cudaStream_t (void*).
 * Asynchronous; launch errors (CUDA) returned. UNSUPPORTED for host-only or
 * row-partitioned handles (use crsd_spmv_dist). x must be finite: a filled
 * zero computes 0*x (as DIA does).
 * Stream order: JIT handles that run as one launch use programmatic dependent
 * launch (CRSD_TUNE_JIT_NO_PDL), so the kernel may start while the previous
 * kernel on `stream` drains, but it reads only the handle's own (immutable)
 * matrix arrays until that kernel has completed; every x / y access is
 * ordered after it, exactly as with a plain launch.
 */
crsd_status_t crsd_spmv(crsd_matrix_t A, const void *alpha, const void *x, const void *beta, void *y,
                        void *stream);

/*
 * End-to-end form with HOST vectors: copies x (and y when beta != 0) to
 * device scratch owned by the handle, runs crsd_spmv, copies y back and
 * synchronises `stream`. x_host dtype[ncols], y_host dtype[nrows] (pinned
 * memory recommended). Synchronous. Used for the e2e measurement (the
 * paper's transfer caveat).
 */
crsd_status_t crsd_spmv_host(crsd_matrix_t A, const void *alpha, const void *x_host, const void *beta,
                             void *y_host, void *stream);

/* ------------------------------------------------------------------------
 * Row-partitioned multi-GPU path (BASELINE.json north_star (3)). Not in the
 * paper (single GPU). Each rank builds a handle over rows [row_begin,
 * row_end) of a square matrix (opts.row_begin/row_end, COO with GLOBAL
 * indices). x is partitioned like the rows. The rank's x lives in a padded
 * DEVICE buffer x_padded[halo_lo + n_local + halo_hi] whose owned part starts
 * at x_padded + halo_lo; the library writes the halos.
 * ---------------------------------------------------------------------- */

/* Halo widths (elements) and local length of a row-partitioned handle.
 * halo_lo is a multiple of 4 so x_padded + halo_lo stays 16-byte aligned. */
crsd_status_t crsd_dist_x_layout(crsd_matrix_t A, int64_t *halo_lo, int64_t *n_local, int64_t *halo_hi);

/* Communicator. id: 128 bytes from crsd_comm_unique_id() on rank 0,
 * broadcast by the caller (e.g. through torch.distributed). Collective over
 * all ranks. The library creates the NCCL communicator and a comm stream. */
crsd_status_t crsd_comm_unique_id(void *id128);
crsd_status_t crsd_comm_init_rank(const void *id128, int rank, int world, int device, crsd_comm_t *out);
/* Destroy a communicator. Collective for peer-memory communicators: every
 * rank calls it; each rank first finishes all its device work, then tells
 * every peer it is done with the peer's region and waits (bounded) for every
 * peer to say the same before unmapping the peers' regions and freeing its
 * own, so no rank frees memory a slower peer still reads or writes. Destroy
 * the handles bound to it (crsd_destroy) after it. */
crsd_status_t crsd_comm_destroy(crsd_comm_t comm);

/*
 * Peer-memory communicator: the library's own transport (csrc/p2p.cu) in
 * place of NCCL for the halo exchange (north_star (3))
 * and the CG's scalar allreduce. Each rank allocates one device region
 * [flags 64 KB | mailbox parity 0 | mailbox parity 1] and exports it with
 * CUDA IPC; after crsd_comm_p2p_open every rank maps every peer's region
 * (NVLink/NVSwitch loads and stores between GPUs; also works for several
 * processes sharing one GPU). The halo moves by our kernels: the sender
 * packs its send slices into its mailbox and raises a flag in each
 * receiver's region; the receiver waits for the flag and pulls the slices
 * from the peer's mailbox straight into the pads of x_padded, then raises a
 * "consumed" flag so the sender may reuse that parity. Epochs live on the
 * device, so the exchange can be captured into a CUDA graph (crsd_cg does).
 * Every wait is bounded (30 s; the environment variable CRSD_P2P_TIMEOUT_S,
 * read once in crsd_comm_init_p2p, overrides it): on
 * timeout the kernel returns and crsd_comm_error reports a non-zero code
 * instead of the GPU hanging.
 *
 *   crsd_comm_init_p2p(rank, world, device, mailbox_bytes, handle64, &c)
 *       mailbox_bytes: capacity per parity, >= the bytes this rank sends per
 *       exchange (slices rounded up to 256 B; crsd_dist_bind_ranges checks).
 *       handle64: HOST 64 bytes out, this rank's cudaIpcMemHandle_t.
 *       world <= 64. Not collective.
 *   crsd_comm_p2p_open(c, handles)
 *       handles: HOST world*64 bytes, every rank's handle in rank order
 *       (allgathered by the caller, e.g. through torch.distributed).
 *       Must be called on every rank after every rank's init.
 *   crsd_dist_bind_ranges(A, c, ranges4)
 *       The bind of crsd_dist_bind with the range table supplied by the
 *       caller: HOST int64[world][4] = every rank's crsd_dist_ranges() row.
 *       Required for peer-memory communicators (crsd_dist_bind returns
 *       INVALID_ARG for them); also accepted with NCCL communicators.
 *   crsd_comm_allreduce_f64(c, dev, n, stream)
 *       In-place sum of n <= 4 DEVICE doubles over all ranks, stream-ordered.
 *       Peer memory: every rank sums the W contributions in rank order, so
 *       all ranks get bit-identical results. NCCL: ncclAllReduce.
 *   crsd_comm_error(c, &err)
 *       Synchronous. err = 0, or 1/2/3/4 when a send / recv / allreduce /
 *       close wait timed out (a peer never arrived); the results are then
 *       invalid. A communicator with err != 0 is poisoned: its kernels skip
 *       their copies and publish nothing, and once crsd_comm_error has seen
 *       the error, crsd_spmv_dist / crsd_comm_allreduce_f64 / crsd_cg on it
 *       return CRSD_ERR_CUDA. Recreate the communicator.
 *   crsd_dist_x_alloc(A, c, &x_padded)
 *       Collective over the ranks of c (peer-memory communicators; A bound
 *       to c). Allocates this rank's padded x (halo_lo + n_local + halo_hi
 *       elements of the dtype, zeroed, owned by A, freed by crsd_destroy) and
 *       maps every peer's. crsd_spmv_dist called with this x_padded moves the
 *       halo as ONE-SIDED PUTS: each rank stores its send slices straight
 *       into the receivers' pads over NVLink (one crossing per halo byte, no
 *       mailbox copy), signals, and the receivers release the pads after
 *       their boundary segments. Any other x_padded uses the two-stage
 *       mailbox path. crsd_cg over a peer-memory communicator uses this
 *       buffer for p. Every rank must stop using it (crsd_comm_destroy, or a
 *       barrier after its last crsd_spmv_dist) before any rank destroys A.
 *       Ranks must allocate for their handles in the same order (one handle
 *       at a time); a peer that allocated for a different row block is
 *       detected and refused (INVALID_ARG). Bounded by the communicator's
 *       wait limit (CUDA error if a peer never arrives).
 */
crsd_status_t crsd_comm_init_p2p(int rank, int world, int device, int64_t mailbox_bytes, void *ipc_handle64,
                                 crsd_comm_t *out);
crsd_status_t crsd_comm_p2p_open(crsd_comm_t comm, const void *ipc_handles);
crsd_status_t crsd_dist_bind_ranges(crsd_matrix_t A_local, crsd_comm_t comm, const int64_t *ranges4);
crsd_status_t crsd_comm_allreduce_f64(crsd_comm_t comm, double *dev, int n, void *stream);
crsd_status_t crsd_comm_error(crsd_comm_t comm, int32_t *err);
crsd_status_t crsd_dist_x_alloc(crsd_matrix_t A_local, crsd_comm_t comm, void **x_padded);
/* This handle's row of the range table: {row_begin, row_end, halo_lo_valid,
 * halo_hi_valid} (the halo widths actually needed, without alignment). */
crsd_status_t crsd_dist_ranges(crsd_matrix_t A_local, int64_t *ranges4);

/* Exchange row ranges and halo widths with every rank (collective, once per
 * handle and communicator) and derive the send/recv plan. */
crsd_status_t crsd_dist_bind(crsd_matrix_t A_local, crsd_comm_t comm, void *stream);

/*
 * Distributed SpMV (north_star (3)): the halo exchange
 * (peer-memory kernels or NCCL send/recv, per the communicator) runs on the
 * communicator's highest-priority stream in parallel with the interior
 * segments on `stream`; the boundary segments follow the exchange on the
 * comm stream (concurrently with the interior; CRSD_TUNE_DIST_BOUNDARY_SERIAL
 * runs them on `stream` after it) and `stream` joins the comm stream before
 * the call returns, so y_local is complete in `stream` order. Asynchronous.
 * With a peer-memory communicator and x_padded from crsd_dist_x_alloc the
 * halo moves as one-sided puts, and (JIT variant) the receive is fused into
 * the boundary kernel: each boundary CTA waits for the senders' flags before
 * copying its x windows and the last one releases the pads
 * (CRSD_TUNE_HALO_UNFUSED: separate wait / release kernels).
 *   x_padded  DEVICE dtype[halo_lo+n_local+halo_hi], 16-byte aligned; the
 *             owned part must be written before the call (stream-ordered);
 *             the halo parts are overwritten.
 *   y_local   DEVICE dtype[n_local].
 * comm == NULL means "halos already filled by the caller": only the compute
 * runs (single-process testing of the partitioned layout).
 */
crsd_status_t crsd_spmv_dist(crsd_matrix_t A_local, const void *alpha, void *x_padded, const void *beta,
                             void *y_local, crsd_comm_t comm, void *stream);

/*
 * Pure host helper (no CUDA, no NCCL): given every rank's [row_begin,
 * row_end, halo_lo_valid, halo_hi_valid] (int64[world][4], the halo widths
 * actually needed, without alignment padding) compute what `rank` receives
 * and sends. Output arrays have capacity `world` entries each:
 *   recv_peer[k], recv_begin[k] (global col), recv_count[k]; *nrecv
 *   send_peer[k], send_begin[k] (global col), send_count[k]; *nsend
 * Multi-hop is handled: a halo wider than a neighbour's block is split over
 * every owner. Errors: INVALID_ARG (ranges not contiguous / not covering).
 */
crsd_status_t crsd_dist_plan(int world, int rank, const int64_t *ranges4, int64_t *recv_peer,
                             int64_t *recv_begin, int64_t *recv_count, int64_t *nrecv, int64_t *send_peer,
                             int64_t *send_begin, int64_t *send_count, int64_t *nsend);

/*
 * Pure host helper: contiguous row blocks aligned to mrows, balanced on
 * per-row weights (e.g. stored bytes per row). weights HOST double[nrows]
 * (NULL => uniform). bounds HOST int64[world+1] receives the row boundaries.
 */
crsd_status_t crsd_partition_rows(int64_t nrows, int32_t mrows, int world, const double *weights,
                                  int64_t *bounds);

/* The paper's scatter-row ELL arrays of a CRSD_PAPER_ELL handle (Fig. 4
 * `num_scatter_rows`, `scatter_rowno`, `num_scatter_width`, `scatter_colval`,
 * `scatter_val`). Two-call protocol: pass NULL
 * arrays to get *nrows_s and *width; then HOST buffers rowno[nrows_s] (global
 * rows), colval[width*nrows_s] and val[width*nrows_s] (dtype), column-major
 * (entry k of row i at k*nrows_s + i), padding col -1 / value 0.
 * UNSUPPORTED if the handle was built without CRSD_PAPER_ELL. */
crsd_status_t crsd_export_paper_ell(crsd_matrix_t A, int64_t *nrows_s, int64_t *width, int64_t *rowno,
                                    int64_t *colval, void *val);

/* Introspection */
crsd_status_t crsd_get_info(crsd_matrix_t A, crsd_info_t *info);
crsd_status_t crsd_export(crsd_matrix_t A, crsd_export_t *out);

/* The CUDA source of the per-pattern codelets the JIT variant compiles for A
 * (the paper's generated codelets): one `case` per distinct
 * pattern with offsets, x windows and shapes as literals. buf (HOST, may be
 * NULL) receives up to cap-1 bytes plus a NUL; *len the full length. Works on
 * host-only handles (no GPU needed). UNSUPPORTED if a segment's staging
 * (values + x windows) exceeds 200 KB of shared memory. */
crsd_status_t crsd_jit_source(crsd_matrix_t A, char *buf, int64_t cap, int64_t *len);

/* The sm_100a cubin NVRTC compiled from crsd_jit_source (compiled here if
 * the handle has none yet; NVRTC only, no GPU needed) -- for inspection with
 * cuobjdump/nvdisasm (the SASS histogram in profiles/). buf (HOST, may be
 * NULL) receives up to cap bytes; *len the full size. UNSUPPORTED without
 * NVRTC or when the staging exceeds 200 KB. */
crsd_status_t crsd_jit_cubin(crsd_matrix_t A, void *buf, int64_t cap, int64_t *len);

/* ------------------------------------------------------------------------
 * Conjugate gradient on a CRSD matrix (the paper
 * motivates CRSD with FDM/FVM coefficient matrices of PDEs, and
 * cites Saad [2], for the iterative methods built on SpMV).
 * Textbook CG (Hestenes & Stiefel; Saad Algorithm 6.18):
 *     r0 = b - A x0; p0 = r0
 *     q = A p; alpha = (r,r)/(p,q); x += alpha p; r -= alpha q;
 *     beta = (r,r)_new/(r,r); p = r + beta p
 * A must be symmetric positive definite (not checked) and square.
 * ---------------------------------------------------------------------- */
typedef struct {
    int32_t iterations; /* CG steps taken */
    int32_t converged;  /* 1 if sqrt((r,r)) <= rtol * sqrt((b,b)) was reached */
    double rr0;         /* (r_0, r_0) */
    double rr;          /* (r_k, r_k) at exit (recurrence residual) */
    double bb;          /* (b, b) */
    int64_t launches;   /* kernel launches of the solve (graph nodes included) */
} crsd_cg_result_t;

/*
 * Solve A x = b.
 *   b          DEVICE dtype[n_local], 16-byte aligned, read-only.
 *   x          DEVICE dtype[n_local], 16-byte aligned: x0 on entry, the
 *              iterate on exit. n_local = nrows for a one-GPU handle, the
 *              owned rows of a row-partitioned handle.
 *   max_iter   >= 0 steps at most.
 *   rtol       stop when sqrt((r,r)) <= rtol * sqrt((b,b)) (0 => run
 *              max_iter steps, or until (r,r) == 0). Evaluated on the device
 *              after every step.
 *   check_every steps per host poll (and per CUDA graph on one GPU); <= 0 => 16.
 *   comm       NULL for a one-GPU handle; the bound communicator of a
 *              row-partitioned handle (halo exchange through crsd_spmv_dist,
 *              dot products as NCCL allreduces).
 *   rr_history HOST double[max_iter+1] or NULL: (r_j, r_j), j = 0..iterations.
 *   res        HOST, may be NULL.
 *   stream     the work is ordered after prior work on `stream`; the call
 *              returns when the solve has finished (it polls the device).
 * Arithmetic: vectors in the matrix dtype; dot products accumulated in fp64
 * and reduced deterministically; alpha, beta in fp64 (applied in the dtype).
 * The handle owns a workspace (3 vectors + O(SMs) scalars) kept between calls.
 * Errors: INVALID_ARG, UNSUPPORTED (not square / host-only), ALLOC, CUDA, NCCL.
 */
crsd_status_t crsd_cg(crsd_matrix_t A, const void *b, void *x, int32_t max_iter, double rtol,
                      int32_t check_every, crsd_comm_t comm, double *rr_history, crsd_cg_result_t *res,
                      void *stream);

/*
 * Runtime autotuning of the kernel variant (the paper
 * leaves such choices to "the property of matrices"). Times
 * y = A x for every variant whose staging fits (LDG, TMA, PIPE, JIT; the JIT
 * codelets are compiled here if needed) over `reps` launches each (<= 0 =>
 * 20, after 3 warm-ups) and makes the fastest the handle's variant.
 *   x, y     DEVICE vectors as for crsd_spmv (y is overwritten).
 *   ms_out   HOST double[5] or NULL: ms_out[v] = mean ms per launch of
 *            variant v (1..4), -1 if not applicable; ms_out[0] = the best.
 *   chosen   HOST or NULL: the variant chosen (CRSD_VARIANT_*).
 * Synchronous. One-GPU (non-partitioned) handles only.
 */
crsd_status_t crsd_autotune(crsd_matrix_t A, const void *x, void *y, int32_t reps, double *ms_out,
                            int32_t *chosen, void *stream);

/*
 * Build-time autotuning: the row-segment height
 * `mrows` shapes the layout itself, so each candidate in
 * mrows_cand[ncand] (HOST; NULL or ncand <= 0 => the default only) is built
 * like crsd_create_from_coo with opts (NULL => defaults; one-GPU handles
 * only), its variant chosen by crsd_autotune on scratch vectors (reps per
 * variant), and the handle with the fastest SpMV is returned in *out; the
 * others are destroyed as soon as they lose. Candidates the GPU path rejects
 * (e.g. mrows not a multiple of 32*RPT) are skipped. ms_out HOST double[ncand]
 * or NULL: best ms per launch of each candidate (-1 if skipped).
 * Synchronous; peak memory = two candidates' device arrays. Errors as
 * crsd_create_from_coo, plus UNSUPPORTED if no candidate is valid.
 */
crsd_status_t crsd_create_autotuned(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row,
                                    const int64_t *col, const void *val, crsd_dtype_t dtype,
                                    const crsd_opts_t *opts, const int32_t *mrows_cand, int32_t ncand,
                                    int32_t reps, crsd_matrix_t *out, double *ms_out);

/* Number of kernel launches the last crsd_spmv / crsd_spmv_dist / crsd_cg call made. */
crsd_status_t crsd_last_launch_count(crsd_matrix_t A, int32_t *count);

#ifdef __cplusplus
}
#endif
#endif /* CRSD_H */
