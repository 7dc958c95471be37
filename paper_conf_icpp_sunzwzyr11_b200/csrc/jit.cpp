// Runtime code generation of per-pattern SpMV codelets (variant JIT).
//
// The paper's mechanism: after
// the matrix is stored in CRSD, a generator emits one `case` of a `switch` per
// diagonal pattern with the index information baked into the code, and the
// kernel is compiled at runtime (OpenCL there, NVRTC here). Only the values
// (and x, y) are read at SpMV time.
//
// The generated kernel has the data movement of the TMA variant (one CTA per
// segment, thread 0 bulk-copies the segment's value block, warp 0 the x
// windows, one mbarrier), but every pattern-dependent quantity is a literal:
// the diagonal count, the window starts/lengths, each diagonal's offset into
// the staged x, the offsets for the guarded edge path. The codelet for a
// pattern is fully unrolled. NVRTC (libnvrtc.so.12) and the CUDA
// driver API are resolved at runtime (dlopen / cudaGetDriverEntryPoint), so
// libcrsd.so loads on machines without them.
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nvrtc.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <sstream>
#include <string>
#include <vector>

#include "crsd_handle.h"
#include "crsd_internal.h"

namespace crsd {

namespace {

struct NvrtcApi {
    bool ok = false;
    std::string err;
    nvrtcResult (*create)(nvrtcProgram *, const char *, const char *, int, const char *const *, const char *const *);
    nvrtcResult (*compile)(nvrtcProgram, int, const char *const *);
    nvrtcResult (*cubin_size)(nvrtcProgram, size_t *);
    nvrtcResult (*cubin)(nvrtcProgram, char *);
    nvrtcResult (*log_size)(nvrtcProgram, size_t *);
    nvrtcResult (*log)(nvrtcProgram, char *);
    nvrtcResult (*destroy)(nvrtcProgram *);
};

struct DriverApi {
    bool ok = false;
    std::string err;
    CUresult (*load)(CUmodule *, const void *);
    CUresult (*get_function)(CUfunction *, CUmodule, const char *);
    CUresult (*launch)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, CUstream,
                       void **, void **);
    CUresult (*set_attr)(CUfunction, CUfunction_attribute, int);
    CUresult (*unload)(CUmodule);
};

NvrtcApi &nvrtc() {
    static NvrtcApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        const char *names[] = {"libnvrtc.so.12", "/usr/local/cuda/lib64/libnvrtc.so.12", "libnvrtc.so"};
        void *h = nullptr;
        for (const char *n : names)
            if ((h = dlopen(n, RTLD_NOW | RTLD_GLOBAL))) break;
        if (!h) {
            api.err = "libnvrtc.so.12 not found";
            return;
        }
#define SYM(field, name)                                         \
    api.field = reinterpret_cast<decltype(api.field)>(dlsym(h, name)); \
    if (!api.field) {                                            \
        api.err = std::string("missing ") + name;                \
        return;                                                  \
    }
        SYM(create, "nvrtcCreateProgram");
        SYM(compile, "nvrtcCompileProgram");
        SYM(cubin_size, "nvrtcGetCUBINSize");
        SYM(cubin, "nvrtcGetCUBIN");
        SYM(log_size, "nvrtcGetProgramLogSize");
        SYM(log, "nvrtcGetProgramLog");
        SYM(destroy, "nvrtcDestroyProgram");
#undef SYM
        api.ok = true;
    });
    return api;
}

DriverApi &driver() {
    static DriverApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        auto get = [&](const char *name, void **fn) {
            cudaDriverEntryPointQueryResult q;
            return cudaGetDriverEntryPoint(name, fn, cudaEnableDefault, &q) == cudaSuccess &&
                   q == cudaDriverEntryPointSuccess && *fn;
        };
        void *p;
        if (!get("cuModuleLoadData", &p)) { api.err = "cuModuleLoadData"; return; }
        api.load = reinterpret_cast<decltype(api.load)>(p);
        if (!get("cuModuleGetFunction", &p)) { api.err = "cuModuleGetFunction"; return; }
        api.get_function = reinterpret_cast<decltype(api.get_function)>(p);
        if (!get("cuLaunchKernel", &p)) { api.err = "cuLaunchKernel"; return; }
        api.launch = reinterpret_cast<decltype(api.launch)>(p);
        if (!get("cuFuncSetAttribute", &p)) { api.err = "cuFuncSetAttribute"; return; }
        api.set_attr = reinterpret_cast<decltype(api.set_attr)>(p);
        if (!get("cuModuleUnload", &p)) { api.err = "cuModuleUnload"; return; }
        api.unload = reinterpret_cast<decltype(api.unload)>(p);
        api.ok = true;
    });
    return api;
}

// Arguments of the generated kernel (mirrored in the generated source).
template <typename T>
struct JitArgs {
    const T *vals;
    const SegDesc *segs;
    const int32_t *seg_list;
    int64_t seg_begin, seg_count;
    const T *x;
    int64_t x_lo, x_hi;
    T *y;
    int64_t nrows;
    const int32_t *scat_row;
    const int64_t *scat_col;
    const T *scat_val;
    const ScatRec *scat_rec;
    T alpha, beta;
    double *dot_part;
    uint32_t *dot_cnt;
    double *dot_out;
};

const char *kPrelude = R"(
typedef long long i64;
typedef unsigned long long u64;
typedef unsigned int u32;
typedef unsigned short u16;
struct SegDesc { i64 val_base; i64 scat_begin; int off_begin; int nscat; u16 flags; u16 ndias; int plan_begin; };
struct __align__(16) ScatRec { i64 col; double val; int row; int pad[3]; };
struct Args { const T *vals; const SegDesc *segs; const int *seg_list; i64 seg_begin, seg_count;
              const T *x; i64 x_lo, x_hi; T *y; i64 nrows;
              const int *scat_row; const i64 *scat_col; const T *scat_val; const ScatRec *scat_rec; T alpha, beta;
              double *dot_part; u32 *dot_cnt; double *dot_out; };
__device__ __forceinline__ u32 su32(const void *p) { return (u32)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void bar_init(u64 *b) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su32(b)) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void bar_expect(u64 *b, u32 n) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su32(b)), "r"(n) : "memory"); }
__device__ __forceinline__ void bar_wait(u64 *b) {
  u32 done = 0;
  while (!done) asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
                             : "=r"(done) : "r"(su32(b)) : "memory"); }
__device__ __forceinline__ void bar_wait_ph(u64 *b, u32 ph) {
  u32 done = 0;
  while (!done) asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                             : "=r"(done) : "r"(su32(b)), "r"(ph) : "memory"); }
__device__ __forceinline__ u64 pol_first() { u64 p; asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ u64 pol_normal() { u64 p; asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ void g2s(void *dst, const void *src, u32 bytes, u64 *b, u64 pol) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
               :: "r"(su32(dst)), "l"(src), "r"(bytes), "r"(su32(b)), "l"(pol) : "memory"); }
)";

}  // namespace

// Generate the codelets of every distinct pattern of A (TMA data movement,
// whole segment per CTA, Q rows per thread).
static std::string generate(const crsd_matrix_s *A, int Q) {
    const HostCRSD &H = A->H;
    const bool f64 = H.dtype == CRSD_R64F;
    const int m = H.mrows, nt = m / Q, es = H.elem;
    const bool scat = H.nscatter() > 0;  // scatter code only for matrices that have scatter points
    // early issue (default; CRSD_JIT_EARLY=0 for the late form): +1-4 % on
    // C2/C3/C4 (sweep20)
    const bool early = !(getenv("CRSD_JIT_EARLY") && atoi(getenv("CRSD_JIT_EARLY")) == 0);
    std::ostringstream o;
    o << "typedef " << (f64 ? "double" : "float") << " T;\n" << kPrelude;
    o << "#define MROWS " << m << "\n#define NT " << nt << "\n#define Q " << Q << "\n";
    // block sum in a fixed order (shuffle tree per warp, then warps in order);
    // the result is valid in thread 0
    o << "__device__ __forceinline__ double blk_sum(double v, double *red) {\n"
         "  for (int k = 16; k; k >>= 1) v += __shfl_down_sync(0xffffffffu, v, k);\n"
         "  __syncthreads();\n  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;\n  __syncthreads();\n"
         "  double b = 0.0;\n  if (threadIdx.x == 0) for (int k = 0; k < NT / 32; ++k) b += red[k];\n  return b;\n}\n";
    // one __device__ codelet per distinct pattern
    // codelets are keyed by the pattern's plan_begin, which is unique per
    // distinct pattern (off_begin is not: a pattern without diagonals shares
    // it with the next pattern)
    std::vector<int32_t> seen;
    for (const Instance &I : H.inst) {
        const int32_t key = A->segdesc[I.first_seg].plan_begin;
        bool dup = false;
        for (int32_t v : seen) dup |= (v == key);
        if (dup) continue;
        seen.push_back(key);
        const int32_t *pl = A->plan.data() + key;
        const int nd = (int)H.ndias(I.pattern), nwin = pl[0];
        const int64_t *offs = H.pat_offsets.data() + H.pat_ptr[I.pattern];
        o << "// pattern offsets:";
        for (int d = 0; d < nd; ++d) o << " " << offs[d];
        o << "\n__device__ __forceinline__ double codelet_" << key
          << "(const Args &a, const SegDesc &D, i64 row0, bool edge, T *vs, u64 *bar, int t) {\n";
        int64_t xb = 0;
        for (int w = 0; w < nwin; ++w) xb += pl[3 + 2 * w];
        o << "  T *xs = vs + " << (int64_t)nd * m << ";\n";
        // a pattern without diagonals (rows holding only scatter points, or
        // nothing) stages nothing: no mbarrier at all
        // Copy issue. early (default): thread 0 initialises the mbarrier and
        // issues every copy (values, then the x windows) before the CTA
        // barrier, and the scatter gathers are issued before it too. Late
        // form (CRSD_JIT_EARLY=0): thread 0 issues the value copy, lane w of
        // warp 0 issues x window w after the CTA barrier.
        std::string sg;
        if (scat) {
            // scatter points are gathered while the bulk copies are in flight:
            // lane l of every warp reads record l of the segment's first 32
            // (row, col, value in one 32-B record); a ballot keeps those whose
            // row belongs to this warp, which alone load x[col]
            sg = "  int g_own = -1; T g_v = T(0), g_x = T(0); unsigned g_mask = 0u;\n"
                 "  if (D.nscat > 0) {\n"
                 "    const int lane = t & 31;\n"
                 "    ScatRec R; R.col = 0; R.val = 0; R.row = 0;\n"
                 "    if (lane < D.nscat) { R = a.scat_rec[D.scat_begin + lane]; g_own = (R.row % NT) * Q + R.row / NT; }\n"
                 "    const bool mine = g_own >= 0 && (g_own / Q) / 32 == t / 32;\n"
                 "    g_mask = __ballot_sync(0xffffffffu, mine);\n"
                 "    if (mine) { g_v = *reinterpret_cast<const T *>(&R.val); g_x = __ldg(a.x + R.col); }\n"
                 "  }\n";
        }
        // a pattern without diagonals (rows holding only scatter points, or
        // nothing) stages nothing: no mbarrier at all
        if (nd) {
            o << "  if (t == 0) { bar_init(bar); bar_expect(bar, " << (int64_t)nd * m * es << "u + (edge ? 0u : "
              << xb * es << "u));\n";
            o << "    g2s(vs, a.vals + D.val_base, " << (int64_t)nd * m * es << "u, bar, pol_first());\n";
            if (early && nwin) {
                o << "    if (!edge) { const u64 pn = pol_normal();\n";
                int64_t base = 0;
                for (int w = 0; w < nwin; ++w) {
                    o << "      g2s(xs + " << base << ", a.x + row0 + (" << pl[2 + 2 * w] << "), "
                      << (int64_t)pl[3 + 2 * w] * es << "u, bar, pn);\n";
                    base += pl[3 + 2 * w];
                }
                o << "    }\n";
            }
            o << "  }\n";
            if (early) o << sg;
            o << "  __syncthreads();\n";
        } else {
            o << "  (void)xs; (void)bar;\n";
            if (early) o << sg;
        }
        if (nwin && !early) {
            o << "  if (!edge && t < 32) { const u64 pn = pol_normal();\n";
            int64_t base = 0;
            for (int w = 0; w < nwin; ++w) {
                o << "    if (t == " << (w % 32) << ") g2s(xs + " << base << ", a.x + row0 + (" << pl[2 + 2 * w] << "), "
                  << (int64_t)pl[3 + 2 * w] * es << "u, bar, pn);\n";
                base += pl[3 + 2 * w];
            }
            o << "  }\n";
        }
        if (!early) o << sg;
        o << "  T acc[Q];\n#pragma unroll\n  for (int q = 0; q < Q; ++q) acc[q] = T(0);\n";
        // fused dot: x[row] is loaded now, while the bulk copies fly, not in
        // the epilogue (a load there would add a memory latency to every CTA)
        o << "  T xr[Q];\n  if (a.dot_part) {\n#pragma unroll\n    for (int q = 0; q < Q; ++q) {\n"
             "      const i64 r = row0 + t + q * NT;\n      xr[q] = (!edge || r < a.nrows) ? __ldg(a.x + r) : T(0);\n    }\n  }\n";
        if (nd) o << "  bar_wait(bar);\n";
        const int32_t *xoff = pl + 2 + 2 * nwin;
        o << "  if (!edge) {\n#pragma unroll\n    for (int q = 0; q < Q; ++q) {\n      const int r = t + q * NT;\n";
        for (int d = 0; d < nd; ++d)
            o << "      acc[q] = fma(vs[" << (int64_t)d * m << " + r], xs[" << xoff[d] << " + r], acc[q]);\n";
        o << "    }\n  } else {\n#pragma unroll\n    for (int q = 0; q < Q; ++q) {\n      const i64 r = row0 + t + q * NT;\n";
        for (int d = 0; d < nd; ++d)
            o << "      { const i64 i = r + (" << offs[d] << "); acc[q] = fma(vs[" << (int64_t)d * m
              << " + t + q * NT], (i >= a.x_lo && i < a.x_hi) ? __ldg(a.x + i) : T(0), acc[q]); }\n";
        o << "    }\n  }\n";
        // scatter points in (row, col) order by their owner thread: the
        // gathered ones (broadcast from the lane holding them), then any
        // beyond the first 32; then the epilogue
        if (scat)
            o << "  if (D.nscat > 0) {\n"
                 "    for (unsigned mm = g_mask; mm; mm &= mm - 1) {\n"
                 "      const int j = __ffs(mm) - 1;\n"
                 "      const int own = __shfl_sync(0xffffffffu, g_own, j);\n"
                 "      const T v = __shfl_sync(0xffffffffu, g_v, j), xv = __shfl_sync(0xffffffffu, g_x, j);\n"
                 "#pragma unroll\n      for (int q = 0; q < Q; ++q) if (own == t * Q + q) acc[q] = fma(v, xv, acc[q]);\n"
                 "    }\n"
                 "    for (int e = 32; e < D.nscat; ++e) {\n"
                 "      const int rr = __ldg(a.scat_row + D.scat_begin + e);\n"
                 "      if (rr % NT != t) continue;\n"
                 "      const T v = __ldg(a.scat_val + D.scat_begin + e), xv = __ldg(a.x + __ldg(a.scat_col + D.scat_begin + e));\n"
                 "#pragma unroll\n      for (int q = 0; q < Q; ++q) if (rr / NT == q) acc[q] = fma(v, xv, acc[q]);\n"
                 "    }\n  }\n";
        // epilogue; with a fused dot (CG: (p, q) with p = x) each thread
        // also accumulates x[row] * y[row] in fp64
        o << "  double dsum = 0.0;\n#pragma unroll\n  for (int q = 0; q < Q; ++q) {\n    const i64 r = row0 + t + q * NT;\n"
             "    if (!edge || r < a.nrows) {\n      T *yp = a.y + r;\n"
             "      const T out = (a.beta != T(0)) ? fma(a.alpha, acc[q], a.beta * *yp) : a.alpha * acc[q];\n"
             "      __stcs(yp, out);\n"
             "      if (a.dot_part) dsum = fma((double)xr[q], (double)out, dsum);\n    }\n"
             "  }\n  return dsum;\n}\n";
    }
    o << "extern \"C\" __global__ void __launch_bounds__(NT) crsd_jit(const Args a) {\n"
         "  extern __shared__ __align__(128) unsigned char smem[];\n  __shared__ u64 bar;\n"
         "  const i64 s = a.seg_list ? (i64)__ldg(a.seg_list + blockIdx.x) : a.seg_begin + blockIdx.x;\n"
         "  const SegDesc D = a.segs[s];\n  const i64 row0 = s * MROWS;\n  const bool edge = (D.flags & 1) != 0;\n"
         "  T *vs = reinterpret_cast<T *>(smem);\n  double d = 0.0;\n  switch (D.plan_begin) {\n";
    for (int32_t v : seen) o << "  case " << v << ": d = codelet_" << v << "(a, D, row0, edge, vs, &bar, threadIdx.x); break;\n";
    o << "  }\n";
    // fused dot, deterministic two-level reduction: every CTA writes its
    // partial; the last CTA to arrive in each group of 256 CTAs sums that
    // group's partials (one load per thread, fixed tree order) into a group
    // partial; the last group sums the group partials. One counter per group
    // keeps the atomics spread and the tail to two short reductions (a single
    // last CTA summing every partial was a ~30 us serial tail per launch).
    o << "  if (a.dot_part) {\n"
         "    __shared__ double red[NT / 32];\n    __shared__ bool last;\n"
         "    const unsigned G = (gridDim.x + 255u) / 256u, g = blockIdx.x / 256u;\n"
         "    const unsigned gs = min(256u, gridDim.x - g * 256u);\n"
         "    double *gpart = a.dot_part + gridDim.x;\n"
         "    d = blk_sum(d, red);\n"
         "    if (threadIdx.x == 0) {\n      a.dot_part[blockIdx.x] = d;\n      __threadfence();\n"
         "      last = atomicAdd(a.dot_cnt + g, 1u) == gs - 1;\n    }\n    __syncthreads();\n"
         "    if (last) {\n      __threadfence();\n"
         "      double b = 0.0;\n"
         "      for (unsigned k = threadIdx.x; k < gs; k += NT) b += __ldcg(a.dot_part + g * 256u + k);\n"
         "      b = blk_sum(b, red);\n"
         "      if (threadIdx.x == 0) {\n        gpart[g] = b;\n        a.dot_cnt[g] = 0u;\n        __threadfence();\n"
         "        last = atomicAdd(a.dot_cnt + G, 1u) == G - 1;\n      }\n      __syncthreads();\n"
         "      if (last) {\n        __threadfence();\n        double c = 0.0;\n"
         "        for (unsigned k = threadIdx.x; k < G; k += NT) c += __ldcg(gpart + k);\n"
         "        c = blk_sum(c, red);\n"
         "        if (threadIdx.x == 0) {\n          *a.dot_out = c;\n          a.dot_cnt[G] = 0u;\n        }\n      }\n    }\n  }\n";
    o << "}\n";
    return o.str();
}

// Persistent, double-buffered form of the codelets (kernel crsd_jitp): a
// CTA per SM slot loops over its segments (w, w + G, ...) with two staging
// buffers. Warp 0 refills a buffer as soon as every thread is done with it:
// lane 0 copies the segment descriptor into the buffer's header and issues
// the bulk copies (values, x windows) with every pattern quantity a literal;
// the 32 lanes read the segment's first 32 scatter records and gather their
// x[col] into the header. The segment after next is therefore in flight
// while the current one computes, and no CTA start-up (launch, descriptor
// load, scatter gather) sits between a buffer's reuse and its next copy.
static void generate_persistent(const crsd_matrix_s *A, int Q, std::ostringstream &o) {
    const HostCRSD &H = A->H;
    const int m = H.mrows, es = H.elem;
    const bool scat = H.nscatter() > 0;
    o << "\n// ---- persistent double-buffered form ----\n"
         "struct __align__(16) StageHdr { SegDesc D; i64 row0; int nsg; int pad; int own[32]; T v[32]; T xv[32]; };\n"
         "#define HDR ((int)((sizeof(StageHdr) + 127) / 128 * 128))\n";
    std::vector<int32_t> seen;
    std::ostringstream issue_sw, comp_sw;
    for (const Instance &I : H.inst) {
        const int32_t key = A->segdesc[I.first_seg].plan_begin;
        bool dup = false;
        for (int32_t v : seen) dup |= (v == key);
        if (dup) continue;
        seen.push_back(key);
        const int32_t *pl = A->plan.data() + key;
        const int nd = (int)H.ndias(I.pattern), nwin = pl[0];
        const int64_t *offs = H.pat_offsets.data() + H.pat_ptr[I.pattern];
        int64_t xb = 0;
        for (int w = 0; w < nwin; ++w) xb += pl[3 + 2 * w];
        // issue (lane 0 of warp 0)
        o << "__device__ __forceinline__ void pissue_" << key
          << "(const Args &a, const SegDesc &D, i64 row0, bool edge, T *vs, u64 *bar) {\n";
        o << "  bar_expect(bar, " << (int64_t)nd * m * es << "u + (edge ? 0u : " << xb * es << "u));\n";
        if (nd) o << "  g2s(vs, a.vals + D.val_base, " << (int64_t)nd * m * es << "u, bar, pol_first());\n";
        if (nwin) {
            o << "  if (!edge) {\n    T *xs = vs + " << (int64_t)nd * m << ";\n    const u64 pn = pol_normal();\n";
            int64_t base = 0;
            for (int w = 0; w < nwin; ++w) {
                o << "    g2s(xs + " << base << ", a.x + row0 + (" << pl[2 + 2 * w] << "), " << (int64_t)pl[3 + 2 * w] * es
                  << "u, bar, pn);\n";
                base += pl[3 + 2 * w];
            }
            o << "  }\n";
        }
        o << "}\n";
        // compute (all threads)
        const int32_t *xoff = pl + 2 + 2 * nwin;
        o << "__device__ __forceinline__ void pcomp_" << key
          << "(const Args &a, const StageHdr &S, bool edge, const T *vs, u64 *bar, u32 ph, int t) {\n";
        o << "  const T *xs = vs + " << (int64_t)nd * m << ";\n  const i64 row0 = S.row0;\n  (void)xs;\n";
        o << "  T acc[Q];\n#pragma unroll\n  for (int q = 0; q < Q; ++q) acc[q] = T(0);\n";
        o << "  bar_wait_ph(bar, ph);\n";
        o << "  if (!edge) {\n#pragma unroll\n    for (int q = 0; q < Q; ++q) {\n      const int r = t + q * NT;\n";
        for (int d = 0; d < nd; ++d)
            o << "      acc[q] = fma(vs[" << (int64_t)d * m << " + r], xs[" << xoff[d] << " + r], acc[q]);\n";
        o << "    }\n  } else {\n#pragma unroll\n    for (int q = 0; q < Q; ++q) {\n      const i64 r = row0 + t + q * NT;\n";
        for (int d = 0; d < nd; ++d)
            o << "      { const i64 i = r + (" << offs[d] << "); acc[q] = fma(vs[" << (int64_t)d * m
              << " + t + q * NT], (i >= a.x_lo && i < a.x_hi) ? __ldg(a.x + i) : T(0), acc[q]); }\n";
        o << "    }\n  }\n";
        if (scat)
            o << "  if (S.D.nscat > 0) {\n"
                 "    for (int e = 0; e < S.nsg; ++e) {\n"
                 "      const int own = S.own[e];\n"
                 "      if (own / Q != t) continue;\n"
                 "#pragma unroll\n      for (int q = 0; q < Q; ++q) if (own == t * Q + q) acc[q] = fma(S.v[e], S.xv[e], acc[q]);\n"
                 "    }\n"
                 "    for (int e = 32; e < S.D.nscat; ++e) {\n"
                 "      const int rr = __ldg(a.scat_row + S.D.scat_begin + e);\n"
                 "      if (rr % NT != t) continue;\n"
                 "      const T v = __ldg(a.scat_val + S.D.scat_begin + e), xv = __ldg(a.x + __ldg(a.scat_col + S.D.scat_begin + e));\n"
                 "#pragma unroll\n      for (int q = 0; q < Q; ++q) if (rr / NT == q) acc[q] = fma(v, xv, acc[q]);\n"
                 "    }\n  }\n";
        o << "#pragma unroll\n  for (int q = 0; q < Q; ++q) {\n    const i64 r = row0 + t + q * NT;\n"
             "    if (!edge || r < a.nrows) { T *yp = a.y + r; __stcs(yp, (a.beta != T(0)) ? fma(a.alpha, acc[q], a.beta * *yp) : a.alpha * acc[q]); }\n"
             "  }\n}\n";
        issue_sw << "      case " << key << ": pissue_" << key << "(a, D, row0, edge, vs, bar); break;\n";
        comp_sw << "    case " << key << ": pcomp_" << key << "(a, S, edge, vk, bar + k, ph, t); break;\n";
    }
    // stage fill by warp 0 (lane = t < 32)
    o << "__device__ __forceinline__ void pfill(const Args &a, i64 w, StageHdr *S, T *vs, u64 *bar, int lane) {\n"
         "  const i64 s = a.seg_list ? (i64)__ldg(a.seg_list + w) : a.seg_begin + w;\n"
         "  const SegDesc D = a.segs[s];\n  const i64 row0 = s * MROWS;\n  const bool edge = (D.flags & 1) != 0;\n"
         "  if (lane == 0) {\n    S->D = D;\n    S->row0 = row0;\n    S->nsg = D.nscat < 32 ? D.nscat : 32;\n"
         "    switch (D.plan_begin) {\n" << issue_sw.str() << "    }\n  }\n";
    if (scat)
        o << "  if (D.nscat > 0 && lane < D.nscat) {\n"
             "    const ScatRec R = a.scat_rec[D.scat_begin + lane];\n"
             "    S->own[lane] = (R.row % NT) * Q + R.row / NT;\n"
             "    S->v[lane] = *reinterpret_cast<const T *>(&R.val);\n"
             "    S->xv[lane] = __ldg(a.x + R.col);\n  }\n";
    o << "}\n";
    o << "extern \"C\" __global__ void __launch_bounds__(NT) crsd_jitp(const Args a, int stage_bytes) {\n"
         "  extern __shared__ __align__(128) unsigned char smem[];\n  __shared__ u64 bar[2];\n"
         "  const int t = threadIdx.x;\n"
         "  if (t == 0) { bar_init(&bar[0]); bar_init(&bar[1]); }\n  __syncthreads();\n"
         "  const i64 G = gridDim.x;\n"
         "  if (t < 32)\n    for (int k = 0; k < 2; ++k) {\n      const i64 w = blockIdx.x + k * G;\n"
         "      unsigned char *b = smem + k * stage_bytes;\n"
         "      if (w < a.seg_count) pfill(a, w, reinterpret_cast<StageHdr *>(b), reinterpret_cast<T *>(b + HDR), bar + k, t);\n    }\n"
         "  __syncthreads();\n"
         "  u32 phs = 0u;  // bit k: phase of buffer k\n  int k = 0;\n"
         "  for (i64 w = blockIdx.x; w < a.seg_count; w += G) {\n"
         "    unsigned char *b = smem + k * stage_bytes;\n"
         "    const StageHdr &S = *reinterpret_cast<const StageHdr *>(b);\n"
         "    const T *vk = reinterpret_cast<const T *>(b + HDR);\n"
         "    const u32 ph = (phs >> k) & 1u;\n"
         "    const bool edge = (S.D.flags & 1) != 0;\n"
         "    switch (S.D.plan_begin) {\n" << comp_sw.str() << "    }\n"
         "    phs ^= 1u << k;\n    __syncthreads();\n"
         "    if (t < 32 && w + 2 * G < a.seg_count)\n"
         "      pfill(a, w + 2 * G, reinterpret_cast<StageHdr *>(b), reinterpret_cast<T *>(b + HDR), bar + k, t);\n"
         "    k ^= 1;\n  }\n}\n";
}

// rows per thread of the generated kernel: <= 256 threads per CTA
static int jit_q(const crsd_matrix_s *A) {
    int q = 1;
    while (A->H.mrows / q > 256) q *= 2;
    return q;
}

// staging buffer of the persistent kernel: header + the largest staging
static int64_t jitp_stage_bytes(const crsd_matrix_s *A) {
    const int64_t hdr = (32 + 8 + 8 + 4 * 32 + 2 * 32 * (int64_t)A->H.elem + 127) / 128 * 128;
    return (hdr + A->smem_bytes + 127) / 128 * 128;
}

std::string jit_generate(const crsd_matrix_s *A) {
    std::string src = generate(A, jit_q(A));
    std::ostringstream o;
    generate_persistent(A, jit_q(A), o);
    return src + o.str();
}

// Range launches on forked streams, concurrently (default), or one after the
// other on the caller's stream (CRSD_JIT_CONCURRENT=0).
static bool jit_concurrent() {
    static const bool v = !(getenv("CRSD_JIT_CONCURRENT") && atoi(getenv("CRSD_JIT_CONCURRENT")) == 0);
    return v;
}

// The kernel's dynamic shared memory is one number per launch, so a single
// launch reserves the LARGEST pattern's staging for every CTA: on C4 the
// 19-diagonal rows (56 KB, 4 CTAs/SM) set the reservation for the 9- and
// 11-diagonal rows too, which alone would fit 7-8 CTAs per SM. Instances are
// contiguous segment ranges, so the one-GPU launch is split into runs of
// instances with the same occupancy class, each launched with its own
// staging size (see below for when it pays). CRSD_JIT_RANGES=0 disables
// the split, =2 forces it at every class change (tests, sanitizer runs).
static void jit_plan_ranges(crsd_matrix_s *A) {
    const HostCRSD &H = A->H;
    A->jit_ranges.clear();
    const int64_t nseg = H.nseg;
    const int64_t nt = H.mrows / jit_q(A);
    const int mode = getenv("CRSD_JIT_RANGES") ? atoi(getenv("CRSD_JIT_RANGES")) : 1;
    const bool off = mode == 0;
    const bool force = mode == 2;  // testing: split at every class change, no folding, no cost rule
    std::vector<int64_t> whole = {0, nseg, A->smem_bytes, 0};
    if (off || H.inst.empty()) {
        A->jit_ranges.push_back(whole);
        return;
    }
    auto staging = [&](const Instance &I) {
        const int32_t *pl = A->plan.data() + A->segdesc[I.first_seg].plan_begin;
        int64_t el = H.ndias(I.pattern) * H.mrows;
        for (int w = 0; w < pl[0]; ++w) el += pl[3 + 2 * w];
        return el * H.elem;
    };
    auto occupancy = [&](int64_t b) {
        const int64_t per_cta = (b + 127) / 128 * 128 + 1024 + 128;  // + driver reserve + static smem
        return std::min<int64_t>(2048 / nt, (228 * 1024) / per_cta);
    };
    std::vector<std::vector<int64_t>> runs;
    int64_t run_occ = -1;
    for (const Instance &I : H.inst) {
        const int64_t b = staging(I), occ = occupancy(b);
        if (!runs.empty() && occ == run_occ) {
            runs.back()[1] = I.first_seg + I.nseg - runs.back()[0];
            runs.back()[2] = std::max(runs.back()[2], b);
        } else {
            runs.push_back({I.first_seg, I.nseg, b});
            run_occ = occ;
        }
    }
    // Runs shorter than a few waves (C3's idle sub-block B2 leaves ~48
    // segments per z-plane; C4 has one-segment transitions between its
    // patterns) would cost a whole launch boundary each: fold each into a
    // neighbour with at least as much staging (that neighbour's class does
    // not change); what cannot be folded becomes an "aux" run, launched on a
    // forked stream alongside the main sequence instead of inside it.
    const int64_t min_run = force ? 0 : 4 * (int64_t)A->sm_count;
    for (bool changed = true; changed;) {
        changed = false;
        for (size_t i = 0; i < runs.size(); ++i) {
            if (runs[i][1] >= min_run) continue;
            size_t into = runs.size();
            if (i > 0 && runs[i - 1][2] >= runs[i][2]) into = i - 1;
            else if (i + 1 < runs.size() && runs[i + 1][2] >= runs[i][2]) into = i + 1;
            if (into == runs.size()) continue;
            runs[into][0] = std::min(runs[into][0], runs[i][0]);
            runs[into][1] += runs[i][1];
            runs.erase(runs.begin() + i);
            changed = true;
            break;
        }
    }
    // main sequence: long runs, equal-class neighbours merged when contiguous
    std::vector<std::vector<int64_t>> merged, aux;
    for (const std::vector<int64_t> &r : runs) {
        if (r[1] < min_run) {
            aux.push_back({r[0], r[1], r[2], 1});
            continue;
        }
        if (!merged.empty() && occupancy(merged.back()[2]) == occupancy(r[2]) &&
            merged.back()[0] + merged.back()[1] == r[0]) {
            merged.back()[1] += r[1];
            merged.back()[2] = std::max(merged.back()[2], r[2]);
        } else {
            merged.push_back({r[0], r[1], r[2], 0});
        }
    }
    const size_t max_runs = force ? 64 : 8;
    if (merged.size() + aux.size() <= 1 || merged.size() > max_runs || aux.size() > max_runs) {
        A->jit_ranges.push_back(whole);
        return;
    }
    // Split only if it pays: the staging bytes that get extra CTA slots,
    // sum over the main runs of nseg * staging * (1 - occ_whole / occ_run),
    // must exceed what the extra launch boundaries cost, taken as one wave
    // of the single launch each (sm_count * occ_whole CTAs of the largest
    // staging). C4 (10^8 rows): ~2 GB gained vs 33 MB per boundary -> split;
    // C3 (idle blocks B1 and B3 only, 16 % of the rows): ~32 MB vs ~130 MB
    // -> one launch (measured: a 5-launch split ran at 0.90 against 0.96,
    // sweep24b).
    const int64_t occ_whole = occupancy(A->smem_bytes);
    double gain = 0.0;
    for (const std::vector<int64_t> &r : merged)
        gain += (double)r[1] * (double)r[2] * (1.0 - (double)occ_whole / (double)occupancy(r[2]));
    const double wave = (double)A->sm_count * (double)occ_whole * (double)A->smem_bytes;
    // Concurrent range launches have no boundary to drain; what a split still
    // costs (launches that do not fully overlap, fork/join) is taken as 3/4
    // of a wave in total -- a threshold fitted to sweep25, not derived: C3
    // f64 gains 30.6 MB against a 33.2 MB wave (0.92) and measured 0.960 ->
    // 1.005 split; C3 f32 (mrows 256) gains 15.3 MB against 33.3 MB (0.46)
    // and measured 1.044 -> 0.992 split, so it stays one launch; C4 f32
    // gains ~2 GB (1.013 -> 1.022 against the sequential split).
    const double boundary_cost = jit_concurrent() ? 0.75 * wave : (double)(merged.size() - 1) * wave;
    if (merged.empty() || (!force && gain <= boundary_cost)) {
        A->jit_ranges.push_back(whole);
        return;
    }
    merged.insert(merged.end(), aux.begin(), aux.end());
    A->jit_ranges = merged;
}

crsd_status_t jit_build(crsd_matrix_s *A) {
    NvrtcApi &nv = nvrtc();
    if (!nv.ok) return fail(CRSD_ERR_UNSUPPORTED, "JIT variant: " + nv.err);
    DriverApi &dr = driver();
    if (!dr.ok) return fail(CRSD_ERR_UNSUPPORTED, "JIT variant: driver entry point " + dr.err);
    if (A->smem_bytes > 200 * 1024) return fail(CRSD_ERR_UNSUPPORTED, "JIT variant: a segment's staging exceeds 200 KB");
    if (A->H.npat() > 256) return fail(CRSD_ERR_UNSUPPORTED, "JIT variant: more than 256 distinct patterns");
    A->jit_source = jit_generate(A);
    nvrtcProgram prog;
    if (nv.create(&prog, A->jit_source.c_str(), "crsd_jit.cu", 0, nullptr, nullptr) != NVRTC_SUCCESS)
        return fail(CRSD_ERR_CUDA, "nvrtcCreateProgram failed");
    const char *opts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-default-device", "-lineinfo"};
    nvrtcResult r = nv.compile(prog, 4, opts);
    if (r != NVRTC_SUCCESS) {
        size_t n = 0;
        nv.log_size(prog, &n);
        std::string log(n, '\0');
        nv.log(prog, &log[0]);
        nv.destroy(&prog);
        return fail(CRSD_ERR_CUDA, "NVRTC compile failed: " + log.substr(0, 2000));
    }
    size_t n = 0;
    nv.cubin_size(prog, &n);
    std::vector<char> cubin(n);
    nv.cubin(prog, cubin.data());
    nv.destroy(&prog);
    CUmodule mod;
    CUfunction fn;
    if (dr.load(&mod, cubin.data()) != CUDA_SUCCESS) return fail(CRSD_ERR_CUDA, "cuModuleLoadData failed");
    if (dr.get_function(&fn, mod, "crsd_jit") != CUDA_SUCCESS) {
        dr.unload(mod);
        return fail(CRSD_ERR_CUDA, "cuModuleGetFunction(crsd_jit) failed");
    }
    if (A->smem_bytes > 48 * 1024 &&
        dr.set_attr(fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)A->smem_bytes) != CUDA_SUCCESS) {
        dr.unload(mod);
        return fail(CRSD_ERR_CUDA, "cuFuncSetAttribute failed");
    }
    // persistent form: usable when two staging buffers fit one CTA
    CUfunction fnp = nullptr;
    const int64_t pbytes = 2 * jitp_stage_bytes(A);
    if (pbytes <= 220 * 1024 && dr.get_function(&fnp, mod, "crsd_jitp") == CUDA_SUCCESS) {
        if (pbytes > 48 * 1024 &&
            dr.set_attr(fnp, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)pbytes) != CUDA_SUCCESS)
            fnp = nullptr;
    } else {
        fnp = nullptr;
    }
    A->jit_module = mod;
    A->jit_function = fn;
    A->jitp_function = fnp;
    jit_plan_ranges(A);
    return CRSD_OK;
}

void jit_free(crsd_matrix_s *A) {
    for (size_t i = 0; i < A->jit_pool.size(); ++i) {
        cudaStreamSynchronize((cudaStream_t)A->jit_pool[i]);
        cudaStreamDestroy((cudaStream_t)A->jit_pool[i]);
        cudaEventDestroy((cudaEvent_t)A->jit_ev_join[i]);
    }
    if (A->jit_ev_fork) cudaEventDestroy((cudaEvent_t)A->jit_ev_fork);
    A->jit_pool.clear();
    A->jit_ev_join.clear();
    A->jit_ev_fork = nullptr;
    if (A->jit_module && driver().ok) driver().unload((CUmodule)A->jit_module);
    A->jit_module = nullptr;
    A->jit_function = nullptr;
    A->jitp_function = nullptr;
}

template <typename T>
int jit_launch(const crsd_matrix_s *A, const SpmvArgs<T> &s, void *stream) {
    if (s.seg_count <= 0) return 0;
    JitArgs<T> j;
    j.vals = s.vals;
    j.segs = s.segs;
    j.seg_list = s.seg_list;
    j.seg_begin = s.seg_begin;
    j.seg_count = s.seg_count;
    j.x = s.x;
    j.x_lo = s.x_lo;
    j.x_hi = s.x_hi;
    j.y = s.y;
    j.nrows = s.nrows;
    j.scat_row = s.scat_row;
    j.scat_col = s.scat_col;
    j.scat_val = s.scat_val;
    j.scat_rec = s.scat_rec;
    j.dot_part = s.dot_part;
    j.dot_cnt = s.dot_cnt;
    j.dot_out = s.dot_out;
    j.alpha = s.alpha;
    j.beta = s.beta;
    const unsigned nt = (unsigned)(A->H.mrows / jit_q(A));
    CUresult r;
    // persistent form (CRSD_JIT_MODE=persist, or A->jit_persist): no fused dot
    const char *mode = getenv("CRSD_JIT_MODE");
    const bool persist = A->jitp_function && !s.dot_part &&
                         (mode ? std::string(mode) == "persist" : A->jit_persist);
    if (persist) {
        int stage = (int)jitp_stage_bytes(A);
        const int64_t per_cta = 2 * (int64_t)stage + 1024 + 64;
        int64_t per_sm = std::min<int64_t>(2048 / nt, (228 * 1024) / per_cta);
        per_sm = std::min<int64_t>(per_sm, 65536 / (32 * (int64_t)nt));
        if (per_sm < 1) per_sm = 1;
        int64_t grid = std::min<int64_t>(s.seg_count, per_sm * A->sm_count);
        void *pp[] = {&j, &stage};
        r = driver().launch((CUfunction)A->jitp_function, (unsigned)grid, 1, 1, nt, 1, 1, (unsigned)(2 * stage),
                            (CUstream)stream, pp, nullptr);
    } else if (!s.seg_list && !s.dot_part && A->jit_ranges.size() > 1) {
        // a segment range (the whole matrix, or a contiguous interior):
        // one launch per occupancy class it meets (jit_plan_ranges)
        // Concurrent mode (default, CRSD_JIT_CONCURRENT=1): every range on
        // its own forked stream, all joined at the end -- the ranges are
        // independent (disjoint rows), so no launch waits for another's
        // drain and their tails overlap. Sequential mode (=0): the main
        // ranges one after the other on `stream`, aux runs on a forked stream.
        int n = 0;
        const int64_t b0 = s.seg_begin, b1 = s.seg_begin + s.seg_count;
        crsd_matrix_s *M = const_cast<crsd_matrix_s *>(A);
        const bool conc = jit_concurrent();
        int next = 0, nstreams = 0;
        auto pool_stream = [&](int i) -> CUstream {
            while ((int)M->jit_pool.size() <= i) {
                cudaStream_t as;
                cudaEvent_t ej;
                if (cudaStreamCreateWithFlags(&as, cudaStreamNonBlocking) != cudaSuccess ||
                    cudaEventCreateWithFlags(&ej, cudaEventDisableTiming) != cudaSuccess)
                    return nullptr;
                M->jit_pool.push_back(as);
                M->jit_ev_join.push_back(ej);
            }
            if (!M->jit_ev_fork) {
                cudaEvent_t ef;
                if (cudaEventCreateWithFlags(&ef, cudaEventDisableTiming) != cudaSuccess) return nullptr;
                M->jit_ev_fork = ef;
            }
            if (i == 0 && cudaEventRecord((cudaEvent_t)M->jit_ev_fork, (cudaStream_t)stream) != cudaSuccess)
                return nullptr;
            if (cudaStreamWaitEvent((cudaStream_t)M->jit_pool[i], (cudaEvent_t)M->jit_ev_fork, 0) != cudaSuccess)
                return nullptr;
            return (CUstream)M->jit_pool[i];
        };
        for (int pass = 0; pass < 2; ++pass) {
            for (const std::vector<int64_t> &rg : A->jit_ranges) {
                if (rg[3] != (pass == 0 ? 1 : 0)) continue;
                const int64_t lo = std::max(b0, rg[0]), hi = std::min(b1, rg[0] + rg[1]);
                if (lo >= hi) continue;
                CUstream st = (CUstream)stream;
                if (conc || rg[3]) {
                    // concurrent: one stream per range (pool of 8, reused
                    // round-robin); sequential: the aux runs share stream 0
                    const int i = conc ? (next++) % 8 : 0;
                    if (i < nstreams) {
                        st = (CUstream)M->jit_pool[i];
                    } else {
                        if ((st = pool_stream(i)) == nullptr) return -(int)cudaErrorLaunchFailure;
                        nstreams = i + 1;
                    }
                }
                j.seg_begin = lo;
                j.seg_count = hi - lo;
                void *params[] = {&j};
                r = driver().launch((CUfunction)A->jit_function, (unsigned)(hi - lo), 1, 1, nt, 1, 1,
                                    (unsigned)rg[2], st, params, nullptr);
                if (r != CUDA_SUCCESS) return -(int)cudaErrorLaunchFailure;
                ++n;
            }
        }
        for (int i = 0; i < nstreams; ++i)
            if (cudaEventRecord((cudaEvent_t)M->jit_ev_join[i], (cudaStream_t)M->jit_pool[i]) != cudaSuccess ||
                cudaStreamWaitEvent((cudaStream_t)stream, (cudaEvent_t)M->jit_ev_join[i], 0) != cudaSuccess)
                return -(int)cudaErrorLaunchFailure;
        return n;
    } else {
        void *params[] = {&j};
        r = driver().launch((CUfunction)A->jit_function, (unsigned)s.seg_count, 1, 1, nt, 1, 1,
                            (unsigned)A->smem_bytes, (CUstream)stream, params, nullptr);
    }
    return r == CUDA_SUCCESS ? 1 : -(int)cudaErrorLaunchFailure;
}

template int jit_launch<double>(const crsd_matrix_s *, const SpmvArgs<double> &, void *);
template int jit_launch<float>(const crsd_matrix_s *, const SpmvArgs<float> &, void *);

}  // namespace crsd

extern "C" crsd_status_t crsd_jit_source(crsd_matrix_t A, char *buf, int64_t cap, int64_t *len) {
    if (!A || !len) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    if (A->smem_bytes > 200 * 1024)
        return crsd::fail(CRSD_ERR_UNSUPPORTED, "JIT codelets need a segment's staging <= 200 KB");
    const std::string src = A->jit_source.empty() ? crsd::jit_generate(A) : A->jit_source;
    *len = (int64_t)src.size();
    if (buf && cap > 0) {
        const int64_t n = std::min<int64_t>(cap - 1, (int64_t)src.size());
        std::memcpy(buf, src.data(), n);
        buf[n] = 0;
    }
    return CRSD_OK;
}
