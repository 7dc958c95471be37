// Internal structures of libcrsd (host builder <-> C-ABI <-> CUDA kernels).
// Not part of the public ABI (include/crsd.h).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "../../include/crsd.h"

namespace crsd {

// NVTX range for profilers (nsys / ncu --nvtx); a no-op without a tool attached.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};

// ----------------------------------------------------------------------------
// errors
// ----------------------------------------------------------------------------
void set_error(const std::string &msg);
crsd_status_t fail(crsd_status_t st, const std::string &msg);

// ----------------------------------------------------------------------------
// Host CRSD (B200 layout)
// ----------------------------------------------------------------------------
struct Instance {          // the paper's diagonal pattern p (Table II)
    int64_t first_seg;     // SR_p / mrows
    int64_t nseg;          // NRS_p
    int32_t pattern;       // index into HostCRSD::pat_*
    int64_t val_base;      // sum_{i<p} NRS_i * NNzRS_i
};

// Segment flags
enum : int32_t { SEG_EDGE = 1, SEG_BOUNDARY = 2 };

// Per-segment descriptor read by one CTA (uniform).
struct alignas(16) SegDesc {
    int64_t val_base;    // slot of (segment, d=0, l=0)
    int64_t scat_begin;  // first scatter entry of the segment
    int32_t off_begin;   // first offset of the segment's pattern in pat_offs
    int32_t nscat;       // scatter entries
    uint16_t flags;      // SEG_*
    uint16_t ndias;      // NDias of the pattern (<= MAX_NDIAS)
    int32_t plan_begin;  // TMA staging plan of the pattern in `plan`
};
constexpr int MAX_NDIAS = 4096;

// Kernel variants
enum : int32_t { VARIANT_AUTO = 0, VARIANT_LDG = 1, VARIANT_TMA = 2, VARIANT_PIPE = 3, VARIANT_JIT = 4 };

// TMA staging plan of one distinct pattern (int32 words at plan_begin):
//   [0] nwin  [1] smem bytes (values + windows)
//   then nwin x (start, count): x window [row0 + start, row0 + start + count)
//        (start, count multiples of 16/sizeof(T) elements)
//   then ndias x xoff: element offset in the smem x region of row 0's x for
//        diagonal d (= window base + o_d - start)
//   then ndias x window index of diagonal d

static_assert(sizeof(SegDesc) == 32, "SegDesc must be 32 bytes");

// Scatter point as one 32-byte record (col relative to the x base, value as
// the matrix dtype in the first bytes of `val`, row within the segment), so a
// segment's points can be staged with one bulk copy (PIPE kernel).
struct alignas(16) ScatRec {
    int64_t col;
    double val;   // float matrices use the first 4 bytes
    int32_t row;
    int32_t pad[3];
};
static_assert(sizeof(ScatRec) == 32, "ScatRec must be 32 bytes");

// Scatter slab (JIT codelets): the first SLAB_K scatter points of segment s
// at slab[s * SLAB_K + l], 16 bytes each, so a CTA loads its points from an
// address it knows without any load (no segment-descriptor round trip before
// the x gathers). Every slot, used or not, carries the segment's point count
// n (saturated at 65535); points beyond SLAB_K are read from the plain
// arrays (scat_row/col/val at scat_begin + l) after the descriptor load.
constexpr int SLAB_K = 16;
struct alignas(16) SlabRec {
    int32_t col;    // column relative to the local x base
    uint16_t row;   // row within the segment
    uint16_t n;     // the segment's scatter points, min(n, 65535)
    double val;     // float matrices use the first 4 bytes
};
static_assert(sizeof(SlabRec) == 16, "SlabRec must be 16 bytes");

struct HostCRSD {
    int64_t nrows = 0, ncols = 0;    // global
    int64_t row_begin = 0, row_end = 0;
    int64_t n_local = 0;             // row_end - row_begin
    bool partitioned = false;
    int32_t mrows = 256, idle_max = 255;
    crsd_dtype_t dtype = CRSD_R64F;
    int elem = 8;                    // sizeof(value)
    int64_t nseg = 0;
    int64_t nnz = 0;

    // distinct patterns (ascending offsets)
    std::vector<int64_t> pat_ptr;     // npat + 1
    std::vector<int64_t> pat_offsets;
    std::vector<Instance> inst;

    std::vector<uint8_t> vals;        // nslots * elem
    int64_t nslots = 0, ndiag_nnz = 0;

    std::vector<int64_t> scat_ptr;    // nseg + 1
    std::vector<int32_t> scat_row;    // row within segment
    std::vector<int64_t> scat_col;    // global column
    std::vector<uint8_t> scat_val;    // nscatter * elem

    // paper-exact scatter rows (flag CRSD_PAPER_ELL): every row
    // holding a scatter point, stored WHOLE in ELL (column-major, ascending
    // columns, col -1 / value 0 padding); the SpMV overwrites those rows
    bool paper_ell = false;
    int64_t ell_nrows = 0, ell_width = 0;
    std::vector<int64_t> ell_rowno;   // local row of each ELL row
    std::vector<int64_t> ell_col;     // ell_width * ell_nrows, global column or -1
    std::vector<uint8_t> ell_val;     // same, dtype

    // column extent actually referenced (global), over stored entries
    int64_t min_col_ref = 0, max_col_ref = -1;

    int64_t npat() const { return (int64_t)pat_ptr.size() - 1; }
    int64_t nscatter() const { return scat_ptr.empty() ? 0 : scat_ptr.back(); }
    int64_t ndias(int32_t p) const { return pat_ptr[p + 1] - pat_ptr[p]; }
};

struct BuildOptions {
    int32_t mrows, idle_max;
    uint32_t flags;
    int64_t row_begin, row_end;
    int32_t nthreads;
};

// COO -> HostCRSD. val points to float or double per dtype.
crsd_status_t build_from_coo(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *row, const int64_t *col,
                             const void *val, crsd_dtype_t dtype, const BuildOptions &o, HostCRSD &H);
crsd_status_t build_from_csr(int64_t nrows, int64_t ncols, const int64_t *row_ptr, const int64_t *col,
                             const void *val, crsd_dtype_t dtype, const BuildOptions &o, HostCRSD &H);

// x window of a segment for the GPU kernel with RPT rows per thread: the
// element range [lo, hi) relative to the local x base that the vector loads
// of a non-edge segment touch.
void segment_x_window(const HostCRSD &H, int64_t s, int rpt, int64_t &lo, int64_t &hi);

// Segment descriptors + flags. x_lo/x_hi: valid x range relative to the
// local x base; own_hi: n_local (the x the rank owns is [0, own_hi)).
void make_segdescs(const HostCRSD &H, int rpt, int64_t x_lo, int64_t x_hi, std::vector<SegDesc> &out);

// TMA staging plans of all distinct patterns (x windows = clusters of offsets
// closer than `gap` elements); fills SegDesc::plan_begin; returns max smem.
int64_t make_plans(const HostCRSD &H, int64_t gap, std::vector<int32_t> &plan, std::vector<SegDesc> &segs,
                   int64_t *xmax_elems = nullptr);

// Halo extents (elements outside [0, n_local) relative to the local x base)
// the handle needs: from its non-edge windows and its scatter columns.
void needed_halo(const HostCRSD &H, int rpt, int64_t &need_lo, int64_t &need_hi);

// ----------------------------------------------------------------------------
// device side
// ----------------------------------------------------------------------------
// Receive side of a one-sided halo exchange fused into the boundary
// segments' kernel (JIT variant, peer-memory direct mode; dist.cpp): every
// CTA's thread 0 waits (bounded) until each sender has published this
// epoch's puts (ready[peer[k]] >= halo_epoch + 1) before it copies x windows
// that reach into the pads; the last CTA to finish releases the pads to the
// senders (*consumed[k] = epoch) and advances halo_epoch. Mirrored in the
// generated source (jit.cpp).
constexpr int HALO_MAX_PEERS = 16;
struct HaloSync {
    const uint64_t *ready;                 // my flags.ready[], indexed by peer rank
    uint64_t *halo_epoch;                  // my flags.halo_epoch
    uint32_t *counter;                     // my flags.counter[1] (grid arrival)
    uint32_t *err;                         // my flags.err (set on timeout)
    uint64_t *consumed[HALO_MAX_PEERS];    // &peer_flags(sender k)->consumed[me]
    int32_t peer[HALO_MAX_PEERS];          // sender ranks
    int32_t npeer, pad_;
    uint64_t timeout_ns;
};

template <typename T>
struct SpmvArgs {
    const T *vals;
    const SegDesc *segs;
    const int32_t *pat_offs;
    const int32_t *plan;
    const int32_t *scat_row;
    const int64_t *scat_col;  // relative to x base
    const T *scat_val;
    const ScatRec *scat_rec;  // same points as 32-byte records
    const SlabRec *scat_slab; // per-segment slab of the first SLAB_K points (JIT), or null
    const T *x;               // local x base (x_padded + halo_lo for dist)
    int64_t x_lo, x_hi;       // valid x range relative to x
    T *y;
    int64_t nrows;            // local rows
    const int32_t *seg_list;  // if non-null: CTA work = seg_list[i]
    int64_t seg_begin, seg_count;
    int32_t mrows;
    int32_t smem_bytes;       // largest whole-segment staging (values + x windows), bytes
    int32_t pipe_xmax_elems;  // PIPE variant: largest x staging of a pattern (elements)
    int32_t max_ndias;        // largest NDias over patterns
    int32_t tma_split;        // TMA variant: CTAs per segment (each covers mrows/split rows)
    int32_t tma_q;            // TMA variant: rows per thread
    int64_t tma_smem;         // TMA variant: dynamic shared memory per CTA
    int32_t has_scatter;      // the matrix has scatter points (selects the staging kernel)
    int32_t variant;          // VARIANT_LDG / _TMA / _PIPE / _JIT
    T alpha, beta;
    const HaloSync *halo = nullptr;  // JIT boundary launch with the fused halo receive, or null
    bool pdl = false;                // JIT: programmatic dependent launch allowed (CRSD_TUNE_JIT_PDL)
};

// Paper-exact scatter rows (CRSD_PAPER_ELL): y[rowno[i]] = alpha * sum_k
// val[k*n+i] * x[col[k*n+i]], ascending k, separately rounded mul and add.
// Returns a cudaError_t value (0 = ok).
template <typename T>
int launch_paper_ell(const int64_t *rowno, const int64_t *col, const T *val, int64_t n, int64_t width, const T *x,
                     T *y, T alpha, void *stream);

// Launch the SpMV kernel for the given work (range or list) on `stream`.
// Returns number of launches (0 if no work) or -1 on launch error.
template <typename T>
int launch_spmv(const SpmvArgs<T> &a, int sm_count, void *stream);

}  // namespace crsd
