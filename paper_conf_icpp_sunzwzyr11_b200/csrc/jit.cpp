// Runtime code generation of per-pattern SpMV codelets (variant JIT).
//
// The paper's mechanism: after
// the matrix is stored in CRSD, a generator emits one `case` of a `switch` per
// diagonal pattern with the index information baked into the code, and the
// kernel is compiled at runtime (OpenCL there, NVRTC here). Only the values
// (and x, y) are read at SpMV time.
//
// The generated kernel runs one CTA per row segment. Thread 0
// bulk-copies (cp.async.bulk, SASS UBLKCP) the segment's value block and its
// x windows into shared memory; every pattern-dependent quantity is a
// literal: the diagonal count, the window starts/lengths, each diagonal's
// offset into the staged x, the offsets for the guarded edge path. The
// codelet for a pattern is fully unrolled.
//
// Staging chunks. The value block and the windows are split into chunks,
// each completing on its own mbarrier (by default one chunk per x window:
// the window and the value runs of the diagonals that read it). The FMAs of
// chunk c start as soon as chunk c has landed while the later chunks are
// still in flight, so a CTA holds its shared memory for less time after its
// last byte arrives than with one barrier for the whole segment.
//
// Descriptor-free issue. The segment -> pattern lookup (the paper's group_id
// -> pattern) is baked into the kernel as a comparison tree over
// the instances' first segments, with each instance's value base as a
// literal, so thread 0 issues the bulk copies without waiting for any memory
// load. A segment's first 16 scatter points come from a fixed-address slab
// (SlabRec), loaded as the CTA's first instruction; only points beyond them
// need the segment descriptor.
//
// Register staging (reg_diags / crsd_jit_rs): where it turns a handle that
// needs occupancy-class range launches into one launch, the values of the
// last diagonals of heavy patterns are loaded into registers instead of
// shared memory, so one more CTA (and its bytes in flight) fits per SM.
//
// Programmatic dependent launch (jit_pdl): one-launch handles let the next
// crsd_spmv's CTAs start during the previous kernel's tail; they stream the
// (immutable) values first and wait (griddepcontrol.wait) before x and y.
//
// NVRTC (libnvrtc.so.12) and the CUDA driver API are resolved at runtime
// (dlopen / cudaGetDriverEntryPoint), so libcrsd.so loads on machines
// without them.
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
    CUresult (*launch_ex)(const CUlaunchConfig *, CUfunction, void **, void **) = nullptr;  // optional (PDL)
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
        if (get("cuLaunchKernelEx", &p)) api.launch_ex = reinterpret_cast<decltype(api.launch_ex)>(p);
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
    const SlabRec *scat_slab;
    T alpha, beta;
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
              const int *scat_row; const i64 *scat_col; const T *scat_val; const ScatRec *scat_rec; const int4 *scat_slab;
              T alpha, beta; };
__device__ __forceinline__ u32 su32(const void *p) { return (u32)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void bar_init(u64 *b) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su32(b)) : "memory"); }
__device__ __forceinline__ void bar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void bar_expect(u64 *b, u32 n) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su32(b)), "r"(n) : "memory"); }
__device__ __forceinline__ void bar_wait(u64 *b) {
  u32 done = 0;
  while (!done) asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
                             : "=r"(done) : "r"(su32(b)) : "memory"); }
__device__ __forceinline__ u64 pol_first() { u64 p; asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ u64 pol_normal() { u64 p; asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p)); return p; }
struct HaloSync { const u64 *ready; u64 *halo_epoch; u32 *counter; u32 *err; u64 *consumed[16]; int peer[16];
                  int npeer, pad_; u64 timeout_ns; };
__device__ __forceinline__ u64 ld_acquire_sys(const u64 *p) {
  u64 v; asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ void st_release_sys(u64 *p, u64 v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory"); }
// thread 0: every sender has published epoch e (bounded wait; err = 2 on timeout);
// then order the async-proxy (bulk copy) reads of the pads after the acquire
__device__ __noinline__ void halo_wait(const HaloSync &h, u64 e) {
  for (int k = 0; k < h.npeer; ++k) {
    const u64 *f = h.ready + h.peer[k];
    if (ld_acquire_sys(f) >= e) continue;
    u64 t0; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    while (ld_acquire_sys(f) < e) {
      __nanosleep(128);
      u64 t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      if (t - t0 > h.timeout_ns) { atomicExch(h.err, 2u); break; }
    }
  }
  asm volatile("fence.proxy.async.global;" ::: "memory");
}
__device__ __forceinline__ void g2s(void *dst, const void *src, u32 bytes, u64 *b, u64 pol) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
               :: "r"(su32(dst)), "l"(src), "r"(bytes), "r"(su32(b)), "l"(pol) : "memory"); }
)";

// One staging chunk: diagonals [d0, d1) of a pattern's value block and,
// when win >= 0, the x window `win` (whose diagonals start at d0).
struct Chunk {
    int d0, d1, win;
};

// Chunks of a pattern. chunk < 0: one chunk (one mbarrier) holding the whole
// value block and every window (win == -2); chunk == 0: one chunk per x
// window (the window's diagonals are contiguous: windows are clusters of
// consecutive offsets, make_plans); chunk > 0: windows further split into
// runs of at most `chunk` diagonals, the window riding with the first.
std::vector<Chunk> make_chunks(const int32_t *pl, int nd, int chunk) {
    std::vector<Chunk> out;
    if (nd == 0) return out;
    if (chunk < 0) {
        out.push_back({0, nd, -2});
        return out;
    }
    const int nwin = pl[0];
    const int32_t *xwin = pl + 2 + 2 * nwin + nd;
    const int step = chunk > 0 ? chunk : nd;
    for (int d = 0; d < nd;) {
        int e = d;
        while (e + 1 < nd && xwin[e + 1] == xwin[d]) ++e;
        for (int a = d; a <= e; a += step) out.push_back({a, std::min(e + 1, a + step), a == d ? xwin[d] : -1});
        d = e + 1;
    }
    return out;
}

// Instances as leaves of the baked segment -> (pattern, value base) lookup.
struct Leaf {
    int64_t first, stride, val_base;
    int32_t key;
};

void emit_locate(std::ostringstream &o, const std::vector<Leaf> &L, size_t lo, size_t hi, int depth) {
    const std::string ind(2 + 2 * depth, ' ');
    if (hi - lo == 1) {
        const Leaf &f = L[lo];
        o << ind << "{ key = " << f.key << "; vb = " << f.val_base << "LL + (s - " << f.first << "LL) * " << f.stride
          << "LL; }\n";
        return;
    }
    const size_t mid = (lo + hi) / 2;
    o << ind << "if (s < " << L[mid].first << "LL) {\n";
    emit_locate(o, L, lo, mid, depth + 1);
    o << ind << "} else {\n";
    emit_locate(o, L, mid, hi, depth + 1);
    o << ind << "}\n";
}

}  // namespace

// Programmatic dependent launch (PDL) for crsd_spmv: a one-GPU handle whose
// matrix runs as one launch. Consecutive SpMVs on a stream then overlap: the
// next launch's CTAs take the SM slots the previous kernel's last wave frees
// and stream their values while it drains (frac of the copy peak, plain ->
// PDL: C2 f64 1.080 -> 1.101, C2 f32 1.054 -> 1.091, C3 f32 1.044 -> 1.069;
// profiles/r02/sweep6_pdl_default.jsonl). Occupancy-class range launches
// keep their concurrent forked streams: a PDL chain of the ranges measured
// 0.89-0.93 against 0.98-1.03 on C3 f64 (sweep5_pdl_chain.jsonl).
bool jit_pdl(const crsd_matrix_s *A) {
    return !(A->tune & CRSD_TUNE_JIT_NO_PDL) && !A->H.partitioned && A->jit_ranges.size() <= 1;
}

// rows per thread of the generated kernel: <= 256 threads per CTA
static int jit_q(const crsd_matrix_s *A) {
    int q = 1;
    while (A->H.mrows / q > 256) q *= 2;
    return q;
}

// Staging bytes (values + x windows) of one CTA of instance I, and the CTAs
// per SM a launch with `b` bytes of dynamic shared memory per CTA allows.
static int64_t staging_smem(const crsd_matrix_s *A, const Instance &I) {
    const HostCRSD &H = A->H;
    const int32_t *pl = A->plan.data() + A->segdesc[I.first_seg].plan_begin;
    int64_t el = H.ndias(I.pattern) * H.mrows;
    for (int w = 0; w < pl[0]; ++w) el += pl[3 + 2 * w];
    return el * H.elem;
}
static int64_t occupancy_of(const crsd_matrix_s *A, int64_t b) {
    const int64_t nt = A->H.mrows / jit_q(A);
    const int64_t per_cta = (b + 127) / 128 * 128 + 1024 + 256;  // + driver reserve + static smem (barriers)
    return std::min<int64_t>(2048 / nt, (228 * 1024) / per_cta);
}
// Register staging (one-GPU handles; jit_decide): the values of the last R
// diagonals of instance I's pattern are loaded by their own threads into
// registers (coalesced streaming loads issued at CTA start) instead of
// staged in shared memory, R just large enough that one more CTA fits per SM
// -- bytes in flight are what the kernel's rate follows and
// shared memory caps them. Such segments run in a second kernel
// (crsd_jit_rs) whose launch bounds give the registers for it.
// Returns R (0: no register staging for this pattern) and the target CTAs
// per SM.
static int reg_diags(const crsd_matrix_s *A, const Instance &I, int64_t *target = nullptr) {
    const HostCRSD &H = A->H;
    if (A->regstage <= 0 || (A->tune & CRSD_TUNE_JIT_NO_REGSTAGE) || H.partitioned) return 0;
    const int Q = jit_q(A), nt = H.mrows / Q, nd = (int)H.ndias(I.pattern);
    const int64_t S = staging_smem(A, I), occ = occupancy_of(A, S), run = (int64_t)H.mrows * H.elem;
    const int64_t tgt = occ + 1;
    if (tgt > 2048 / nt) return 0;
    const int64_t cap = ((228 * 1024) / tgt - 1024 - 256) / 128 * 128;
    const int64_t R = (S - cap + run - 1) / run;
    if (R <= 0 || R > nd) return 0;
    // registers: ~32 for the codelet itself plus R * Q values (two per fp64)
    const int64_t allowed = (65536 / (tgt * nt)) / 8 * 8;
    if (32 + R * Q * (H.elem / 4) > allowed) return 0;
    if (target) *target = tgt;
    return (int)R;
}
static int64_t inst_staging(const crsd_matrix_s *A, const Instance &I) {
    return staging_smem(A, I) - (int64_t)reg_diags(A, I) * A->H.mrows * A->H.elem;
}
// the register-staged kernel's CTAs per SM (0: no instance uses it)
static int64_t rs_min_blocks(const crsd_matrix_s *A) {
    int64_t mb = 0;
    for (const Instance &I : A->H.inst) {
        int64_t t = 0;
        if (reg_diags(A, I, &t) > 0) mb = std::max(mb, t);
    }
    return mb;
}

// [a, b) runs of edge segments
static std::vector<std::pair<int64_t, int64_t>> edge_runs(const crsd_matrix_s *A) {
    std::vector<std::pair<int64_t, int64_t>> edges;
    for (int64_t s = 0; s < A->H.nseg; ++s)
        if (A->segdesc[s].flags & SEG_EDGE) {
            if (!edges.empty() && edges.back().second == s) edges.back().second = s + 1;
            else edges.push_back({s, s + 1});
        }
    return edges;
}
// the generated kernel carries the baked segment -> (pattern, value base) lookup
static bool jit_locate(const crsd_matrix_s *A, const std::vector<std::pair<int64_t, int64_t>> &edges) {
    return !(A->tune & CRSD_TUNE_JIT_DESC_ISSUE) && !A->H.inst.empty() && A->H.inst.size() <= 4096 &&
           edges.size() <= 16;
}

// Generate the codelets of every distinct pattern of A (one CTA per segment,
// Q rows per thread) and the kernel that dispatches to them.
static std::string generate(const crsd_matrix_s *A, int Q) {
    const HostCRSD &H = A->H;
    const bool f64 = H.dtype == CRSD_R64F;
    const int m = H.mrows, nt = m / Q, es = H.elem;
    const bool scat = H.nscatter() > 0;  // scatter code only for matrices that have scatter points
    // programmatic dependent launch (jit_pdl): the value copies (the matrix
    // never changes) are issued before griddepcontrol.wait, the x windows,
    // scatter gathers and y after it
    const bool pdl = jit_pdl(A);
    // scatter slab: a CTA's first SLAB_K points from a fixed address
    const bool slab = scat && slab_ok(A);
    std::ostringstream o;
    o << "typedef " << (f64 ? "double" : "float") << " T;\n" << kPrelude;
    // a slab record's value (int4 .z/.w): the dtype's bits, no local-memory round trip
    o << (f64 ? "#define SLAB_VAL(r) __hiloint2double((r).w, (r).z)\n" : "#define SLAB_VAL(r) __int_as_float((r).z)\n");
    o << "#define MROWS " << m << "\n#define NT " << nt << "\n#define Q " << Q << "\n";
    // one __device__ codelet per distinct pattern, keyed by the pattern's
    // plan_begin (unique per distinct pattern; off_begin is not: a pattern
    // without diagonals shares it with the next pattern)
    std::vector<int32_t> seen;
    int nbar = 1;
    for (const Instance &I : H.inst) {
        const int32_t key = A->segdesc[I.first_seg].plan_begin;
        bool dup = false;
        for (int32_t v : seen) dup |= (v == key);
        if (dup) continue;
        seen.push_back(key);
        const int32_t *pl = A->plan.data() + key;
        const int nd = (int)H.ndias(I.pattern), nwin = pl[0];
        const int64_t *offs = H.pat_offsets.data() + H.pat_ptr[I.pattern];
        const int32_t *xoff = pl + 2 + 2 * nwin;
        std::vector<int64_t> wbase(nwin + 1, 0);
        for (int w = 0; w < nwin; ++w) wbase[w + 1] = wbase[w] + pl[3 + 2 * w];
        const std::vector<Chunk> ch = make_chunks(pl, nd, A->jit_chunk);
        nbar = std::max(nbar, (int)ch.size());
        o << "// pattern offsets:";
        for (int d = 0; d < nd; ++d) o << " " << offs[d];
        o << "\n// " << ch.size() << " staging chunk(s)\n";
        // halo (compile-time after inlining): the crsd_jit_halo kernel, whose
        // x windows and scatter gathers may reach into pads written by the
        // neighbours' one-sided puts -- thread 0 issues the value copies,
        // waits for the senders, then issues the window copies; the scatter
        // gathers move after the CTA barrier
        // pass 0: the codelet; pass 1 (register staging, reg_diags > 0): the
        // same codelet with the values of the last R diagonals loaded into
        // registers by their own threads instead of staged in shared memory
        const int rdiag = reg_diags(A, I);
        for (int pass = 0; pass < (rdiag > 0 ? 2 : 1); ++pass) {
        const int R = pass ? rdiag : 0, ns = nd - R;  // ns diagonals staged in shared memory
        o << "__device__ __forceinline__ void codelet_" << (pass ? "rs_" : "") << key
          << "(const Args &a, const i64 s, const i64 vb, const i64 row0, const bool edge, T *vs, u64 *bar, const int t,"
             " const bool halo, const HaloSync &hs, const u64 he) {\n";
        if (slab)
            // the slab load needs no other load: issued first, it lands while
            // thread 0 sets up the copies (the matrix never changes, so it may
            // also precede griddepcontrol.wait)
            o << "  int4 sr = make_int4(0, 0, 0, 0);\n"
                 "  if ((t & 31) < " << SLAB_K << ") sr = __ldg(a.scat_slab + s * " << SLAB_K << " + (t & 31));\n";
        if (nd) {
            // thread 0: every mbarrier, then every copy, chunk by chunk
            o << "  T *xs = vs + " << (int64_t)ns * m << ";\n";
            o << "  if (t == 0) {\n";
            for (size_t c = 0; c < ch.size(); ++c) o << "    bar_init(bar + " << c << ");\n";
            o << "    bar_fence_init();\n    const u64 pf = pol_first(), pn = pol_normal();\n";
            for (size_t c = 0; c < ch.size(); ++c) {
                const Chunk &k = ch[c];
                const int64_t vbytes = (int64_t)std::max(0, std::min(k.d1, ns) - k.d0) * m * es;
                int64_t xbytes = 0;
                if (k.win == -2) xbytes = wbase[nwin] * es;
                else if (k.win >= 0) xbytes = (int64_t)pl[3 + 2 * k.win] * es;
                o << "    bar_expect(bar + " << c << ", " << vbytes << "u" << (xbytes ? " + (edge ? 0u : " : "")
                  << (xbytes ? std::to_string(xbytes) + "u)" : "") << ");\n";
                if (vbytes)
                    o << "    g2s(vs + " << (int64_t)k.d0 * m << ", a.vals + vb + " << (int64_t)k.d0 * m << ", " << vbytes
                      << "u, bar + " << c << ", pf);\n";
                if (xbytes && !pdl) {
                    o << "    if (!edge && !halo) {\n";
                    for (int w = 0; w < nwin; ++w) {
                        if (!(k.win == -2 || k.win == w)) continue;
                        o << "      g2s(xs + " << wbase[w] << ", a.x + row0 + (" << pl[2 + 2 * w] << "), "
                          << (int64_t)pl[3 + 2 * w] * es << "u, bar + " << c << ", pn);\n";
                    }
                    o << "    }\n";
                }
            }
            // fused halo receive: the windows after the senders' flags
            o << "    if (halo) {\n      halo_wait(hs, he);\n";
            for (size_t c = 0; c < ch.size(); ++c) {
                const Chunk &k = ch[c];
                if (k.win == -1) continue;
                for (int w = 0; w < nwin; ++w) {
                    if (!(k.win == -2 || k.win == w)) continue;
                    o << "      if (!edge) g2s(xs + " << wbase[w] << ", a.x + row0 + (" << pl[2 + 2 * w] << "), "
                      << (int64_t)pl[3 + 2 * w] * es << "u, bar + " << c << ", pn);\n";
                }
            }
            o << "    }\n";
            o << "  }\n";
            // register-staged values: coalesced streaming loads of the last R
            // diagonals, issued before anything waits (the matrix never changes)
            for (int d = ns; d < nd; ++d)
                o << "  T rv" << d << "[Q];\n#pragma unroll\n  for (int q = 0; q < Q; ++q) rv" << d
                  << "[q] = __ldcs(a.vals + vb + " << (int64_t)d * m << " + t + q * NT);\n";
            if (pdl) {
                // every thread orders its x / y accesses after the previous
                // kernel on the stream; then thread 0 issues the windows
                o << "  if (!halo) {\n    asm volatile(\"griddepcontrol.wait;\" ::: \"memory\");\n"
                     "    if (t == 0 && !edge) {\n      const u64 pn = pol_normal();\n";
                for (size_t c = 0; c < ch.size(); ++c) {
                    const Chunk &k = ch[c];
                    if (k.win == -1) continue;
                    for (int w = 0; w < nwin; ++w) {
                        if (!(k.win == -2 || k.win == w)) continue;
                        o << "      g2s(xs + " << wbase[w] << ", a.x + row0 + (" << pl[2 + 2 * w] << "), "
                          << (int64_t)pl[3 + 2 * w] * es << "u, bar + " << c << ", pn);\n";
                    }
                }
                o << "    }\n  }\n";
            }
        } else {
            o << "  (void)vs; (void)bar; (void)vb;\n";
            o << "  if (halo) { if (t == 0) halo_wait(hs, he); __syncthreads(); }\n";
            if (pdl) o << "  if (!halo) asm volatile(\"griddepcontrol.wait;\" ::: \"memory\");\n";
        }
        if (slab) {
            o << "  int g_own = -1; T g_v = T(0), g_x = T(0); unsigned g_mask = 0u;\n"
                 "  const int nscat = __shfl_sync(0xffffffffu, (sr.y >> 16) & 0xffff, 0);\n";
        } else if (scat) {
            // scatter points are gathered while the bulk copies are in flight:
            // lane l of every warp reads record l of the segment's first 32
            // (row, col, value in one 32-B record); a ballot keeps those whose
            // row belongs to this warp, which alone load x[col]
            o << "  const SegDesc *Dp = a.segs + s;\n  const int nscat = __ldg(&Dp->nscat);\n"
                 "  const i64 sbeg = nscat > 0 ? __ldg(&Dp->scat_begin) : 0;\n"
                 "  int g_own = -1; T g_v = T(0), g_x = T(0); unsigned g_mask = 0u;\n";
        }
        static_assert(SLAB_K == 16, "the generated slab gather assumes 16 slots");
        const char *gather =
            slab ? "  if (nscat > 0) {\n"
                   "    const int lane = t & 31, row = sr.y & 0xffff;\n"
                   "    if (lane < min(nscat, 16)) g_own = (row % NT) * Q + row / NT;\n"
                   "    const bool mine = g_own >= 0 && (g_own / Q) / 32 == t / 32;\n"
                   "    g_mask = __ballot_sync(0xffffffffu, mine);\n"
                   "    if (mine) { g_v = SLAB_VAL(sr); g_x = __ldg(a.x + sr.x); }\n"
                   "  }\n"
                 :
            "  if (nscat > 0) {\n"
            "    const int lane = t & 31;\n"
            "    ScatRec R; R.col = 0; R.val = 0; R.row = 0;\n"
            "    if (lane < nscat) { R = a.scat_rec[sbeg + lane]; g_own = (R.row % NT) * Q + R.row / NT; }\n"
            "    const bool mine = g_own >= 0 && (g_own / Q) / 32 == t / 32;\n"
            "    g_mask = __ballot_sync(0xffffffffu, mine);\n"
            "    if (mine) { g_v = *reinterpret_cast<const T *>(&R.val); g_x = __ldg(a.x + R.col); }\n"
            "  }\n";
        if (scat) o << "  if (!halo) {\n" << gather << "  }\n";
        if (nd) o << "  __syncthreads();\n";
        if (scat) o << "  if (halo) {\n" << gather << "  }\n";
        o << "  T acc[Q];\n#pragma unroll\n  for (int q = 0; q < Q; ++q) acc[q] = T(0);\n";
        // FMAs chunk by chunk, each after its own barrier; ascending offset
        // order within and across chunks (the order of the paper's codelet)
        o << "  if (!edge) {\n";
        for (size_t c = 0; c < ch.size(); ++c) {
            o << "    bar_wait(bar + " << c << ");\n#pragma unroll\n    for (int q = 0; q < Q; ++q) {\n      const int r = t + q * NT;\n";
            for (int d = ch[c].d0; d < ch[c].d1; ++d)
                o << "      acc[q] = fma(" << (d < ns ? "vs[" + std::to_string((int64_t)d * m) + " + r]" : "rv" + std::to_string(d) + "[q]")
                  << ", xs[" << xoff[d] << " + r], acc[q]);\n";
            o << "    }\n";
        }
        o << "  } else {\n";
        for (size_t c = 0; c < ch.size(); ++c) {
            o << "    bar_wait(bar + " << c << ");\n#pragma unroll\n    for (int q = 0; q < Q; ++q) {\n      const i64 r = row0 + t + q * NT;\n";
            for (int d = ch[c].d0; d < ch[c].d1; ++d)
                o << "      { const i64 i = r + (" << offs[d] << "); acc[q] = fma("
                  << (d < ns ? "vs[" + std::to_string((int64_t)d * m) + " + t + q * NT]" : "rv" + std::to_string(d) + "[q]")
                  << ", (i >= a.x_lo && i < a.x_hi) ? __ldg(a.x + i) : T(0), acc[q]); }\n";
            o << "    }\n";
        }
        o << "  }\n";
        // scatter points in (row, col) order by their owner thread: the
        // gathered ones (broadcast from the lane holding them), then any
        // beyond the first 32 (16 with the slab, after the descriptor load);
        // then the epilogue
        if (scat)
            o << "  if (nscat > 0) {\n"
                 "    for (unsigned mm = g_mask; mm; mm &= mm - 1) {\n"
                 "      const int j = __ffs(mm) - 1;\n"
                 "      const int own = __shfl_sync(0xffffffffu, g_own, j);\n"
                 "      const T v = __shfl_sync(0xffffffffu, g_v, j), xv = __shfl_sync(0xffffffffu, g_x, j);\n"
                 "#pragma unroll\n      for (int q = 0; q < Q; ++q) if (own == t * Q + q) acc[q] = fma(v, xv, acc[q]);\n"
                 "    }\n"
              << (slab ? "    if (nscat > 16) {\n"
                         "    const SegDesc *Dp = a.segs + s;\n"
                         "    const int nall = __ldg(&Dp->nscat);\n    const i64 sbeg = __ldg(&Dp->scat_begin);\n"
                         "    for (int e = 16; e < nall; ++e) {\n"
                       : "    {\n    for (int e = 32; e < nscat; ++e) {\n")
              << "      const int rr = __ldg(a.scat_row + sbeg + e);\n"
                 "      if (rr % NT != t) continue;\n"
                 "      const T v = __ldg(a.scat_val + sbeg + e), xv = __ldg(a.x + __ldg(a.scat_col + sbeg + e));\n"
                 "#pragma unroll\n      for (int q = 0; q < Q; ++q) if (rr / NT == q) acc[q] = fma(v, xv, acc[q]);\n"
                 "    }\n    }\n  }\n";
        // epilogue: y = alpha*acc + beta*y, y not read when beta == 0
        o << "#pragma unroll\n  for (int q = 0; q < Q; ++q) {\n    const i64 r = row0 + t + q * NT;\n"
             "    if (!edge || r < a.nrows) {\n      T *yp = a.y + r;\n"
             "      __stcs(yp, (a.beta != T(0)) ? fma(a.alpha, acc[q], a.beta * *yp) : a.alpha * acc[q]);\n    }\n"
             "  }\n}\n";
        }  // pass
    }
    // Baked segment -> (pattern, value base) lookup and edge test, used for
    // range launches (the one-GPU path and contiguous interiors); list
    // launches read the descriptor. Off with CRSD_TUNE_JIT_DESC_ISSUE, or when
    // the tables would be large.
    std::vector<std::pair<int64_t, int64_t>> edges = edge_runs(A);
    const bool locate = jit_locate(A, edges);
    o << "#define NBAR " << nbar << "\n";
    if (locate) {
        std::vector<Leaf> L;
        for (const Instance &I : H.inst)
            L.push_back({I.first_seg, H.ndias(I.pattern) * m, I.val_base, A->segdesc[I.first_seg].plan_begin});
        o << "__device__ __forceinline__ void locate(const i64 s, int &key, i64 &vb) {\n";
        emit_locate(o, L, 0, L.size(), 0);
        o << "}\n__device__ __forceinline__ bool is_edge(const i64 s) {\n  return false";
        for (const auto &e : edges) o << " || (s >= " << e.first << "LL && s < " << e.second << "LL)";
        o << ";\n}\n";
    }
    // the dispatch body shared by crsd_jit and crsd_jit_halo
    o << "__device__ __forceinline__ void run_segment(const Args &a, const bool halo, const HaloSync &hs, const u64 he) {\n"
         "  extern __shared__ __align__(128) unsigned char smem[];\n  __shared__ u64 bar[NBAR];\n"
         "  T *vs = reinterpret_cast<T *>(smem);\n  i64 s, vb;\n  int key;\n  bool edge;\n";
    if (locate)
        o << "  if (!a.seg_list) {\n    s = a.seg_begin + blockIdx.x;\n    locate(s, key, vb);\n    edge = is_edge(s);\n"
             "  } else {\n";
    else
        o << "  {\n";
    o << "    s = a.seg_list ? (i64)__ldg(a.seg_list + blockIdx.x) : a.seg_begin + blockIdx.x;\n"
         "    const SegDesc D = a.segs[s];\n    key = D.plan_begin;\n    vb = D.val_base;\n    edge = (D.flags & 1) != 0;\n"
         "  }\n  const i64 row0 = s * MROWS;\n  switch (key) {\n";
    for (int32_t v : seen)
        o << "  case " << v << ": codelet_" << v << "(a, s, vb, row0, edge, vs, bar, threadIdx.x, halo, hs, he); break;\n";
    o << "  }\n}\n";
    o << "extern \"C\" __global__ void __launch_bounds__(NT) crsd_jit(const Args a) {\n";
    if (pdl) o << "  asm volatile(\"griddepcontrol.launch_dependents;\");\n";
    o << "  const HaloSync hs{};\n  run_segment(a, false, hs, 0ull);\n}\n";
    // register staging: the same dispatch into the register-staged codelets,
    // launch bounds for its CTAs per SM (range launches, baked lookup)
    const int64_t rsb = locate ? rs_min_blocks(A) : 0;
    if (rsb > 0) {
        o << "extern \"C\" __global__ void __launch_bounds__(NT, " << rsb << ") crsd_jit_rs(const Args a) {\n";
        if (pdl) o << "  asm volatile(\"griddepcontrol.launch_dependents;\");\n";
        o << "  extern __shared__ __align__(128) unsigned char smem[];\n  __shared__ u64 bar[NBAR];\n"
             "  T *vs = reinterpret_cast<T *>(smem);\n  const HaloSync hs{};\n  i64 vb;\n  int key;\n"
             "  const i64 s = a.seg_begin + blockIdx.x;\n  locate(s, key, vb);\n  const bool edge = is_edge(s);\n"
             "  const i64 row0 = s * MROWS;\n  switch (key) {\n";
        for (const Instance &I : H.inst) {
            const int32_t key = A->segdesc[I.first_seg].plan_begin;
            bool first = true;
            for (const Instance &J : H.inst)
                if (&J != &I && A->segdesc[J.first_seg].plan_begin == key && &J < &I) first = false;
            if (!first) continue;
            o << "  case " << key << ": codelet_" << (reg_diags(A, I) > 0 ? "rs_" : "") << key
              << "(a, s, vb, row0, edge, vs, bar, threadIdx.x, false, hs, 0ull); break;\n";
        }
        o << "  }\n}\n";
    }
    // boundary segments of a direct-mode exchange: the receive side fused in
    // (wait per CTA before the window copies; the last CTA to finish releases
    // the pads to the senders and advances the epoch)
    o << "extern \"C\" __global__ void __launch_bounds__(NT) crsd_jit_halo(const Args a, const HaloSync hs) {\n"
         "  const u64 he = *(volatile u64 *)hs.halo_epoch + 1;\n"
         "  run_segment(a, true, hs, he);\n"
         "  __shared__ bool last;\n  __threadfence();\n  __syncthreads();\n"
         "  if (threadIdx.x == 0) {\n    last = atomicAdd(hs.counter, 1u) == gridDim.x - 1;\n"
         "    if (last) {\n      *hs.counter = 0u;\n      __threadfence_system();\n"
         "      if (*(volatile u32 *)hs.err == 0u)\n        for (int k = 0; k < hs.npeer; ++k) st_release_sys(hs.consumed[k], he);\n"
         "      *(volatile u64 *)hs.halo_epoch = he;\n    }\n  }\n}\n";
    return o.str();
}

std::string jit_generate(const crsd_matrix_s *A) { return generate(A, jit_q(A)); }

// Range launches on forked streams, concurrently (default), or one after the
// other on the caller's stream (CRSD_TUNE_JIT_SEQUENTIAL).
static bool jit_concurrent(const crsd_matrix_s *A) { return !(A->tune & CRSD_TUNE_JIT_SEQUENTIAL); }

// The kernel's dynamic shared memory is one number per launch, so a single
// launch reserves the LARGEST pattern's staging for every CTA: on C4 the
// 19-diagonal rows (56 KB, 4 CTAs/SM) set the reservation for the 9- and
// 11-diagonal rows too, which alone would fit 7-8 CTAs per SM. Instances are
// contiguous segment ranges, so the one-GPU launch is split into runs of
// instances with the same occupancy class, each launched with its own
// staging size (see below for when it pays). CRSD_TUNE_JIT_ONE_LAUNCH
// disables the split, CRSD_TUNE_JIT_SPLIT_ALL forces it at every class
// change (tests, sanitizer runs).
static void jit_plan_ranges_impl(crsd_matrix_s *A) {
    const HostCRSD &H = A->H;
    A->jit_ranges.clear();
    const int64_t nseg = H.nseg;
    const bool off = (A->tune & CRSD_TUNE_JIT_ONE_LAUNCH) != 0;
    const bool force = (A->tune & CRSD_TUNE_JIT_SPLIT_ALL) != 0;
    int64_t smax = 0;
    for (const Instance &I : H.inst) smax = std::max(smax, inst_staging(A, I));
    if (H.inst.empty()) smax = A->smem_bytes;
    std::vector<int64_t> whole = {0, nseg, smax, 0};
    if (off || H.inst.empty()) {
        A->jit_ranges.push_back(whole);
        return;
    }
    auto staging = [&](const Instance &I) { return inst_staging(A, I); };
    auto occupancy = [&](int64_t b) { return occupancy_of(A, b); };
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
    const int64_t occ_whole = occupancy(smax);
    double gain = 0.0;
    for (const std::vector<int64_t> &r : merged)
        gain += (double)r[1] * (double)r[2] * (1.0 - (double)occ_whole / (double)occupancy(r[2]));
    const double wave = (double)A->sm_count * (double)occ_whole * (double)smax;
    // Concurrent range launches have no boundary to drain; what a split still
    // costs (launches that do not fully overlap, fork/join) is taken as 3/4
    // of a wave in total -- a threshold fitted to sweep25, not derived: C3
    // f64 gains 30.6 MB against a 33.2 MB wave (0.92) and measured 0.960 ->
    // 1.005 split; C3 f32 (mrows 256) gains 15.3 MB against 33.3 MB (0.46)
    // and measured 1.044 -> 0.992 split, so it stays one launch; C4 f32
    // gains ~2 GB (1.013 -> 1.022 against the sequential split).
    const double boundary_cost = jit_concurrent(A) ? 0.75 * wave : (double)(merged.size() - 1) * wave;
    if (merged.empty() || (!force && gain <= boundary_cost)) {
        A->jit_ranges.push_back(whole);
        return;
    }
    merged.insert(merged.end(), aux.begin(), aux.end());
    A->jit_ranges = merged;
}

// ... and mark each range that holds a register-staged instance (element 4):
// it launches crsd_jit_rs.
static void jit_plan_ranges(crsd_matrix_s *A) {
    jit_plan_ranges_impl(A);
    for (std::vector<int64_t> &rg : A->jit_ranges) {
        int64_t rs = 0;
        for (const Instance &I : A->H.inst)
            if (I.first_seg < rg[0] + rg[1] && rg[0] < I.first_seg + I.nseg && reg_diags(A, I) > 0) rs = 1;
        rg.push_back(rs);
    }
}

// Launch plan and register staging: register staging is kept where it turns
// a handle that needs occupancy-class range launches into ONE launch (C3
// f64: its heavy and light instances then all run at 4-5 CTAs per SM, and
// the single launch gets PDL; 1.018 vs 1.002 for the 5 concurrent ranges,
// profiles/r02/sweep12_regstage*.jsonl); where the split remains (C4) it
// measured 1% slower and is not used.
static void jit_decide(crsd_matrix_s *A) {
    // the register-staged kernel dispatches through the baked lookup
    A->regstage = (A->tune & CRSD_TUNE_JIT_NO_REGSTAGE) || A->H.partitioned || !jit_locate(A, edge_runs(A)) ? 0 : 1;
    jit_plan_ranges(A);
    if (A->regstage && (A->jit_ranges.size() > 1 || rs_min_blocks(A) == 0)) {
        A->regstage = 0;
        jit_plan_ranges(A);
    }
}

// Generate and compile A's codelets for sm_100a (NVRTC only; no device needed).
static crsd_status_t jit_compile(crsd_matrix_s *A) {
    NvrtcApi &nv = nvrtc();
    if (!nv.ok) return fail(CRSD_ERR_UNSUPPORTED, "JIT variant: " + nv.err);
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
    A->jit_cubin.resize(n);
    nv.cubin(prog, A->jit_cubin.data());
    nv.destroy(&prog);
    return CRSD_OK;
}

crsd_status_t jit_build(crsd_matrix_s *A) {
    DriverApi &dr = driver();
    if (!dr.ok) return fail(CRSD_ERR_UNSUPPORTED, "JIT variant: driver entry point " + dr.err);
    jit_decide(A);  // before generating: PDL and register staging depend on the launch plan
    crsd_status_t st = jit_compile(A);
    if (st) return st;
    CUmodule mod;
    CUfunction fn;
    if (dr.load(&mod, A->jit_cubin.data()) != CUDA_SUCCESS) return fail(CRSD_ERR_CUDA, "cuModuleLoadData failed");
    if (dr.get_function(&fn, mod, "crsd_jit") != CUDA_SUCCESS) {
        dr.unload(mod);
        return fail(CRSD_ERR_CUDA, "cuModuleGetFunction(crsd_jit) failed");
    }
    if (A->smem_bytes > 48 * 1024 &&
        dr.set_attr(fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)A->smem_bytes) != CUDA_SUCCESS) {
        dr.unload(mod);
        return fail(CRSD_ERR_CUDA, "cuFuncSetAttribute failed");
    }
    CUfunction fh = nullptr;
    if (dr.get_function(&fh, mod, "crsd_jit_halo") != CUDA_SUCCESS ||
        (A->smem_bytes > 48 * 1024 &&
         dr.set_attr(fh, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)A->smem_bytes) != CUDA_SUCCESS)) {
        dr.unload(mod);
        return fail(CRSD_ERR_CUDA, "crsd_jit_halo: cuModuleGetFunction / cuFuncSetAttribute failed");
    }
    CUfunction frs = nullptr;
    if (rs_min_blocks(A) > 0 &&
        (dr.get_function(&frs, mod, "crsd_jit_rs") != CUDA_SUCCESS ||
         (A->smem_bytes > 48 * 1024 &&
          dr.set_attr(frs, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)A->smem_bytes) != CUDA_SUCCESS))) {
        dr.unload(mod);
        return fail(CRSD_ERR_CUDA, "crsd_jit_rs: cuModuleGetFunction / cuFuncSetAttribute failed");
    }
    A->jit_module = mod;
    A->jit_function = fn;
    A->jit_halo_function = fh;
    A->jit_rs_function = frs;

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
    A->jit_halo_function = nullptr;
    A->jit_rs_function = nullptr;
}

// One launch of fn; pdl: with the programmatic-stream-serialization
// attribute (the kernel may start while the previous kernel on the stream
// drains; the codelets wait for it with griddepcontrol.wait).
static CUresult launch_fn(CUfunction fn, unsigned grid, unsigned nt, unsigned smem, CUstream st, void **params,
                          bool pdl) {
    if (!pdl) return driver().launch(fn, grid, 1, 1, nt, 1, 1, smem, st, params, nullptr);
    CUlaunchAttribute at[1];
    std::memset(at, 0, sizeof(at));
    at[0].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
    at[0].value.programmaticStreamSerializationAllowed = 1;
    CUlaunchConfig cfg;
    std::memset(&cfg, 0, sizeof(cfg));
    cfg.gridDimX = grid;
    cfg.gridDimY = cfg.gridDimZ = 1;
    cfg.blockDimX = nt;
    cfg.blockDimY = cfg.blockDimZ = 1;
    cfg.sharedMemBytes = smem;
    cfg.hStream = st;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return driver().launch_ex(&cfg, fn, params, nullptr);
}

template <typename T>
int jit_launch(const crsd_matrix_s *A, const SpmvArgs<T> &s, void *stream) {
    if (s.seg_count <= 0) return 0;
    // PDL only where the codelets were generated for it (jit_pdl: one
    // launch per SpMV), never under stream capture (graph batches keep plain
    // launches)
    bool pdl = s.pdl && !s.halo && !s.seg_list && jit_pdl(A) && driver().launch_ex;
    if (pdl) {
        cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
        if (cudaStreamIsCapturing((cudaStream_t)stream, &cs) != cudaSuccess || cs != cudaStreamCaptureStatusNone)
            pdl = false;
    }
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
    j.scat_slab = s.scat_slab;
    j.alpha = s.alpha;
    j.beta = s.beta;
    const unsigned nt = (unsigned)(A->H.mrows / jit_q(A));
    if (s.halo) {
        // boundary segments with the fused halo receive: one launch
        static_assert(sizeof(HaloSync) == 8 * 4 + 8 * HALO_MAX_PEERS + 4 * HALO_MAX_PEERS + 8 + 8, "HaloSync layout");
        void *params[] = {&j, const_cast<HaloSync *>(s.halo)};
        const CUresult r = driver().launch((CUfunction)A->jit_halo_function, (unsigned)s.seg_count, 1, 1, nt, 1, 1,
                                           (unsigned)A->smem_bytes, (CUstream)stream, params, nullptr);
        return r == CUDA_SUCCESS ? 1 : -(int)cudaErrorLaunchFailure;
    }
    if (!s.seg_list && A->jit_ranges.size() > 1) {
        // a segment range (the whole matrix, or a contiguous interior):
        // one launch per occupancy class it meets (jit_plan_ranges).
        // Concurrent mode (default): every range on its own forked stream,
        // all joined at the end -- the ranges are independent (disjoint
        // rows), so no launch waits for another's drain and their tails
        // overlap. Sequential mode (CRSD_TUNE_JIT_SEQUENTIAL): the main
        // ranges one after the other on `stream`, aux runs on a forked stream.
        int n = 0;
        const int64_t b0 = s.seg_begin, b1 = s.seg_begin + s.seg_count;
        crsd_matrix_s *M = const_cast<crsd_matrix_s *>(A);
        const bool conc = jit_concurrent(A);
        int next = 0, nstreams = 0;
        auto pool_stream = [&](int i) -> CUstream {
            while ((int)M->jit_pool.size() <= i) {
                cudaStream_t as;
                cudaEvent_t ej;
                if (cudaStreamCreateWithFlags(&as, cudaStreamNonBlocking) != cudaSuccess) return nullptr;
                if (cudaEventCreateWithFlags(&ej, cudaEventDisableTiming) != cudaSuccess) {
                    cudaStreamDestroy(as);
                    return nullptr;
                }
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
        // join every forked stream used so far back into `stream` (also on
        // the error path, so later work on `stream` -- or a graph capture --
        // stays ordered after the launches already made)
        auto join = [&]() -> bool {
            bool ok = true;
            for (int i = 0; i < nstreams; ++i)
                ok &= cudaEventRecord((cudaEvent_t)M->jit_ev_join[i], (cudaStream_t)M->jit_pool[i]) == cudaSuccess &&
                      cudaStreamWaitEvent((cudaStream_t)stream, (cudaEvent_t)M->jit_ev_join[i], 0) == cudaSuccess;
            return ok;
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
                        if ((st = pool_stream(i)) == nullptr) {
                            join();
                            return -(int)cudaErrorLaunchFailure;
                        }
                        nstreams = i + 1;
                    }
                }
                j.seg_begin = lo;
                j.seg_count = hi - lo;
                void *params[] = {&j};
                const bool rs = rg.size() > 4 && rg[4] && A->jit_rs_function;
                if (launch_fn((CUfunction)(rs ? A->jit_rs_function : A->jit_function), (unsigned)(hi - lo), nt,
                              (unsigned)rg[2], st, params, false) != CUDA_SUCCESS) {
                    join();
                    return -(int)cudaErrorLaunchFailure;
                }
                ++n;
            }
        }
        return join() ? n : -(int)cudaErrorLaunchFailure;
    }
    void *params[] = {&j};
    // one range over a one-GPU handle: its own kernel and staging size
    // (register staging); lists and row-partitioned handles: the plain kernel
    const bool one = !s.seg_list && A->jit_ranges.size() == 1;
    const bool rs = one && A->jit_ranges[0].size() > 4 && A->jit_ranges[0][4] && A->jit_rs_function;
    const CUresult r = launch_fn((CUfunction)(rs ? A->jit_rs_function : A->jit_function), (unsigned)s.seg_count, nt,
                                 (unsigned)(one ? A->jit_ranges[0][2] : A->smem_bytes), (CUstream)stream, params, pdl);
    return r == CUDA_SUCCESS ? 1 : -(int)cudaErrorLaunchFailure;
}

template int jit_launch<double>(const crsd_matrix_s *, const SpmvArgs<double> &, void *);
template int jit_launch<float>(const crsd_matrix_s *, const SpmvArgs<float> &, void *);

}  // namespace crsd

extern "C" crsd_status_t crsd_jit_source(crsd_matrix_t A, char *buf, int64_t cap, int64_t *len) {
    if (!A || !len) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    if (A->smem_bytes > 200 * 1024)
        return crsd::fail(CRSD_ERR_UNSUPPORTED, "JIT codelets need a segment's staging <= 200 KB");
    if (A->jit_source.empty() && A->jit_ranges.empty()) crsd::jit_decide(A);  // host-only handles: plan as on a device
    const std::string src = A->jit_source.empty() ? crsd::jit_generate(A) : A->jit_source;
    *len = (int64_t)src.size();
    if (buf && cap > 0) {
        const int64_t n = std::min<int64_t>(cap - 1, (int64_t)src.size());
        std::memcpy(buf, src.data(), n);
        buf[n] = 0;
    }
    return CRSD_OK;
}

extern "C" crsd_status_t crsd_jit_cubin(crsd_matrix_t A, void *buf, int64_t cap, int64_t *len) {
    if (!A || !len) return crsd::fail(CRSD_ERR_INVALID_ARG, "NULL argument");
    if (A->jit_cubin.empty()) {
        if (A->jit_ranges.empty()) crsd::jit_decide(A);
        const crsd_status_t st = crsd::jit_compile(A);
        if (st) return st;
    }
    *len = (int64_t)A->jit_cubin.size();
    if (buf && cap > 0) std::memcpy(buf, A->jit_cubin.data(), std::min<int64_t>(cap, *len));
    return CRSD_OK;
}
