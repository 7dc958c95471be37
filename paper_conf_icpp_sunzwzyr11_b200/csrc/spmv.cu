// CRSD SpMV kernels for sm_100a (B200): y = alpha*A*x + beta*y.
//
// Work decomposition (§III-B): one CTA per row segment,
// RPT consecutive rows per thread (RPT = 2 fp64 / 4 fp32) so every value and
// x access is one 128-bit vector. A CTA reads its segment descriptor once,
// which selects the diagonal pattern -- the paper's group_id -> pattern lookup
// precomputed on the host -- so all threads of a CTA take the
// same path. The pattern's offsets come from a small table
// (uniform, L1-resident); no per-nonzero index is loaded.
//
// Per diagonal d (ascending offset o_d):
//   value  vals[val_base + d*mrows + l]     -- 128-bit, coalesced, streamed
//          with an L2 evict_first policy (read exactly once)
//   x      x[row0 + l + o_d]: the thread loads the ALIGNED vector holding
//          x[row0 + RPT*(t + floor(o_d/RPT))]; when o_d is not a multiple of
//          RPT the next vector comes from the neighbour lane by a warp
//          shuffle (lane 31 loads it). This replaces the paper's local-memory
//          staging of x for adjacent groups (Fig. 5) by register
//          exchange: no shared memory, no barrier (the barrier cost the paper
//          measures on wang3/wang4, does not exist here).
//   acc_j = fma(value_j, x_j, acc_j)         -- ascending offset order
// Edge segments (x window outside the valid range, or the partial last
// segment, R9/R11) run a guarded scalar-x body.
// Scatter points of the segment (R5) are added by their owner
// thread after the diagonal part, in (row, col) order; then the epilogue
// writes y once (y read only when beta != 0).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <mutex>

#include "crsd_internal.h"

namespace crsd {

template <typename T>
struct VecT;
template <>
struct VecT<double> {
    using type = double2;
    static constexpr int R = 2;
    static constexpr int LOG = 1;
};
template <>
struct VecT<float> {
    using type = float4;
    static constexpr int R = 4;
    static constexpr int LOG = 2;
};

__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// streamed values: no L1 allocation, L2 evict_first
__device__ __forceinline__ double2 ld_stream(const double2 *ptr, uint64_t pol) {
    double2 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;"
                 : "=d"(r.x), "=d"(r.y)
                 : "l"(ptr), "l"(pol));
    return r;
}
__device__ __forceinline__ float4 ld_stream(const float4 *ptr, uint64_t pol) {
    float4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
                 : "l"(ptr), "l"(pol));
    return r;
}
// x: reused across diagonals (L1) and segments (L2)
__device__ __forceinline__ double2 ld_x(const double2 *ptr) { return __ldg(ptr); }
__device__ __forceinline__ float4 ld_x(const float4 *ptr) { return __ldg(ptr); }

__device__ __forceinline__ void st_stream(double2 *ptr, double2 v) {
    asm volatile("st.global.L1::no_allocate.v2.f64 [%0], {%1, %2};" ::"l"(ptr), "d"(v.x), "d"(v.y) : "memory");
}
__device__ __forceinline__ void st_stream(float4 *ptr, float4 v) {
    asm volatile("st.global.L1::no_allocate.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(ptr), "f"(v.x), "f"(v.y), "f"(v.z),
                 "f"(v.w)
                 : "memory");
}

__device__ __forceinline__ double2 shfl_down1(double2 v) {
    return make_double2(__shfl_down_sync(0xffffffffu, v.x, 1), __shfl_down_sync(0xffffffffu, v.y, 1));
}
__device__ __forceinline__ float4 shfl_down1(float4 v) {
    return make_float4(__shfl_down_sync(0xffffffffu, v.x, 1), __shfl_down_sync(0xffffffffu, v.y, 1),
                       __shfl_down_sync(0xffffffffu, v.z, 1), __shfl_down_sync(0xffffffffu, v.w, 1));
}

__device__ __forceinline__ double get(const double2 &v, int j) { return j == 0 ? v.x : v.y; }
__device__ __forceinline__ float get(const float4 &v, int j) {
    return j == 0 ? v.x : (j == 1 ? v.y : (j == 2 ? v.z : v.w));
}

// x_j = concat(a, b)[al + j], al in [1, R): uniform al, register-only selects
__device__ __forceinline__ void window(const double2 &a, const double2 &b, int /*al == 1*/, double (&xs)[2]) {
    xs[0] = a.y;
    xs[1] = b.x;
}
__device__ __forceinline__ void window(const float4 &a, const float4 &b, int al, float (&xs)[4]) {
    if (al == 1) {
        xs[0] = a.y; xs[1] = a.z; xs[2] = a.w; xs[3] = b.x;
    } else if (al == 2) {
        xs[0] = a.z; xs[1] = a.w; xs[2] = b.x; xs[3] = b.y;
    } else {
        xs[0] = a.w; xs[1] = b.x; xs[2] = b.y; xs[3] = b.z;
    }
}

__device__ __forceinline__ double2 make_vec(const double (&v)[2]) { return make_double2(v[0], v[1]); }
__device__ __forceinline__ float4 make_vec(const float (&v)[4]) { return make_float4(v[0], v[1], v[2], v[3]); }

template <typename T, int CH>
__global__ void __launch_bounds__(256, sizeof(T) == 8 ? 3 : 4) crsd_spmv_ldg(const SpmvArgs<T> a) {
    using V = typename VecT<T>::type;
    constexpr int R = VecT<T>::R;
    constexpr int LOG = VecT<T>::LOG;
    const int t = threadIdx.x;
    const int lane = t & 31;
    const int64_t vstride = a.mrows >> LOG;  // vectors per diagonal of a segment
    const uint64_t pol = policy_evict_first();

    for (int64_t w = blockIdx.x; w < a.seg_count; w += gridDim.x) {
        const int64_t s = a.seg_list ? (int64_t)__ldg(a.seg_list + w) : a.seg_begin + w;
        const SegDesc D = a.segs[s];
        const int64_t row0 = s * a.mrows;
        const int nd = D.ndias;
        const int32_t *offs = a.pat_offs + D.off_begin;
        const V *vb = reinterpret_cast<const V *>(a.vals + D.val_base) + t;
        T acc[R];
#pragma unroll
        for (int j = 0; j < R; ++j) acc[j] = T(0);

        if (!(D.flags & SEG_EDGE)) {
            const V *xv = reinterpret_cast<const V *>(a.x + row0) + t;
            for (int d0 = 0; d0 < nd; d0 += CH) {
                V val[CH], xa[CH], xe[CH];
                int o[CH];
#pragma unroll
                for (int c = 0; c < CH; ++c) {
                    if (d0 + c < nd) {
                        o[c] = __ldg(offs + d0 + c);
                        val[c] = ld_stream(vb + (int64_t)(d0 + c) * vstride, pol);
                    }
                }
#pragma unroll
                for (int c = 0; c < CH; ++c) {
                    if (d0 + c < nd) {
                        const int k = o[c] >> LOG;  // floor(o / R)
                        xa[c] = ld_x(xv + k);
                        if ((o[c] & (R - 1)) && lane == 31) xe[c] = ld_x(xv + k + 1);
                    }
                }
#pragma unroll
                for (int c = 0; c < CH; ++c) {
                    if (d0 + c < nd) {
                        const int al = o[c] & (R - 1);  // warp-uniform
                        T xs[R];
                        if (al == 0) {
#pragma unroll
                            for (int j = 0; j < R; ++j) xs[j] = get(xa[c], j);
                        } else {
                            V nb = shfl_down1(xa[c]);
                            if (lane == 31) nb = xe[c];
                            window(xa[c], nb, al, xs);
                        }
#pragma unroll
                        for (int j = 0; j < R; ++j) acc[j] = fma(get(val[c], j), xs[j], acc[j]);
                    }
                }
            }
        } else {
            // guarded body: x indices outside [x_lo, x_hi) belong to filled
            // zeros only (R9/R11) and are never dereferenced
            const int64_t r = row0 + (int64_t)t * R;
            for (int d = 0; d < nd; ++d) {
                const int o = __ldg(offs + d);
                const V v = ld_stream(vb + (int64_t)d * vstride, pol);
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int64_t idx = r + j + o;
                    const T xj = (idx >= a.x_lo && idx < a.x_hi) ? __ldg(a.x + idx) : T(0);
                    acc[j] = fma(get(v, j), xj, acc[j]);
                }
            }
        }

        // scatter points of this segment, (row, col) order, owner thread adds
        if (D.nscat > 0) {
            const int lo = t * R, hi = lo + R;
            const int32_t *sr = a.scat_row + D.scat_begin;
            int64_t e = 0;
            const int64_t ne = D.nscat;
            if (ne > 32) {  // binary search for the first entry of this thread's rows
                int64_t l = 0, h = ne;
                while (l < h) {
                    const int64_t mid = (l + h) >> 1;
                    if (__ldg(sr + mid) < lo) l = mid + 1; else h = mid;
                }
                e = l;
            }
            for (; e < ne; ++e) {
                const int rr = __ldg(sr + e);
                if (rr >= hi) {
                    if (ne > 32) break;
                    continue;
                }
                if (rr < lo) continue;
                const T v = __ldg(a.scat_val + D.scat_begin + e);
                const T xv = __ldg(a.x + __ldg(a.scat_col + D.scat_begin + e));
#pragma unroll
                for (int j = 0; j < R; ++j)
                    if (rr - lo == j) acc[j] = fma(v, xv, acc[j]);
            }
        }

        // epilogue: y = alpha*acc + beta*y, y not read when beta == 0
        const T al = a.alpha, be = a.beta;
        if (!(D.flags & SEG_EDGE)) {
            V *yv = reinterpret_cast<V *>(a.y + row0) + t;
            T out[R];
            if (be != T(0)) {
                const V yo = *yv;
#pragma unroll
                for (int j = 0; j < R; ++j) out[j] = fma(al, acc[j], be * get(yo, j));
            } else {
#pragma unroll
                for (int j = 0; j < R; ++j) out[j] = al * acc[j];
            }
            st_stream(yv, make_vec(out));
        } else {
            const int64_t r = row0 + (int64_t)t * R;
#pragma unroll
            for (int j = 0; j < R; ++j) {
                if (r + j < a.nrows) {
                    a.y[r + j] = (be != T(0)) ? fma(al, acc[j], be * a.y[r + j]) : al * acc[j];
                }
            }
        }
    }
}

// ---------------------------------------------------------------------------
// TMA-staged variant. One elected thread issues bulk copies
// (cp.async.bulk, Blackwell/Hopper TMA engine) of the segment's contiguous
// value block and of the pattern's x windows (clusters of nearby offsets =
// the paper's adjacent groups) into shared memory, completing on
// one mbarrier; all threads then compute from shared memory. Memory-level
// parallelism no longer depends on registers: a CTA has its whole segment in
// flight (values + x), several CTAs per SM. Thread t owns rows t + q*T
// (T = threads, q < RPT) so shared-memory reads are bank-conflict free.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx_only(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t phase) {
    uint32_t done = 0;
    const uint32_t a = smem_u32(bar);
    while (!done) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(a), "r"(phase)
            : "memory");
    }
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_normal() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
    return p;
}


// A CTA covers `rc` rows of one segment (rc = mrows / split): with split > 1
// the segment's value block is fetched as one bulk copy per diagonal (its rc
// consecutive values), so big segments (many diagonals) still leave several
// CTAs resident per SM. Thread t owns rows t + q*(rc/Q), q < Q.
template <typename T, int Q, bool SCAT>
__global__ void __launch_bounds__(256) crsd_spmv_tma(const SpmvArgs<T> a, int split) {
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t bar;
    const int t = threadIdx.x;
    const int T_ = blockDim.x;
    const int rc = a.mrows / split;  // rows of this CTA
    const int64_t cta = blockIdx.x;
    const int64_t w = split == 1 ? cta : cta / split;
    const int h = split == 1 ? 0 : (int)(cta - w * split);
    const int64_t s = a.seg_list ? (int64_t)__ldg(a.seg_list + w) : a.seg_begin + w;
    const SegDesc D = a.segs[s];
    const int64_t row0 = s * a.mrows + (int64_t)h * rc;
    const int nd = D.ndias;
    const int32_t *plan = a.plan + D.plan_begin;
    const int nwin = __ldg(plan);
    const bool edge = (D.flags & SEG_EDGE) != 0;
    const int shrink = a.mrows - rc;  // each window is this much shorter than for a full segment
    T *vs = reinterpret_cast<T *>(smem);
    T *xs = vs + (int64_t)nd * rc;
    const uint32_t vbytes = (uint32_t)nd * (uint32_t)rc * sizeof(T);
    if (t == 0) {
        mbar_init(&bar, 1);
        mbar_fence_init();
        // plan[1] = values + x bytes of a full segment
        const uint32_t xfull = (uint32_t)__ldg(plan + 1) - (uint32_t)nd * (uint32_t)a.mrows * sizeof(T);
        const uint32_t xbytes = edge ? 0u : xfull - (uint32_t)(nwin * shrink) * sizeof(T);
        mbar_expect_tx(&bar, vbytes + xbytes);
        if (split == 1 && vbytes) bulk_g2s(vs, a.vals + D.val_base, vbytes, &bar, policy_evict_first());
    }
    __syncthreads();
    if (t < 32) {
        // warp 0 issues the remaining copies: one per diagonal of a row slice,
        // one per x window (window q by lane q % 32)
        if (split > 1) {
            const uint64_t pf = policy_evict_first();
            for (int d = t; d < nd; d += 32)
                bulk_g2s(vs + (int64_t)d * rc, a.vals + D.val_base + (int64_t)d * a.mrows + (int64_t)h * rc,
                         (uint32_t)rc * sizeof(T), &bar, pf);
        }
        if (!edge) {
            const uint64_t pn = policy_evict_normal();
            int64_t base = 0;
            for (int q0 = 0; q0 < nwin; q0 += 32) {
                const int q = q0 + t;
                const int st = q < nwin ? __ldg(plan + 2 + 2 * q) : 0;
                const int cnt = q < nwin ? __ldg(plan + 3 + 2 * q) - shrink : 0;
                int inc = cnt;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const int v = __shfl_up_sync(0xffffffffu, inc, o);
                    if (t >= o) inc += v;
                }
                if (q < nwin) bulk_g2s(xs + base + inc - cnt, a.x + row0 + st, (uint32_t)cnt * sizeof(T), &bar, pn);
                base += __shfl_sync(0xffffffffu, inc, 31);
            }
        }
    }
    // Scatter points are gathered now, while the bulk copies are in flight:
    // each warp takes the segment's first 32 entries (lane l -> entry l) and
    // keeps, by ballot, those owned by its threads (owner of local row l is
    // thread l % T_, slot l / T_); entries beyond 32 are read at the end.
    const int lane = t & 31;
    int g_own = -1;
    T g_v = T(0), g_x = T(0);
    unsigned g_mask = 0u;
    if (SCAT && D.nscat > 0) {
        if (lane < D.nscat) {
            const int rr = __ldg(a.scat_row + D.scat_begin + lane) - h * rc;
            if (rr >= 0 && rr < rc) g_own = (rr % T_) * Q + rr / T_;
        }
        const bool mine = g_own >= 0 && (g_own / Q) / 32 == t / 32;
        g_mask = __ballot_sync(0xffffffffu, mine);
        if (mine) {
            g_v = __ldg(a.scat_val + D.scat_begin + lane);
            g_x = __ldg(a.x + __ldg(a.scat_col + D.scat_begin + lane));
        }
    }
    T acc[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) acc[q] = T(0);
    const int32_t *xoff = plan + 2 + 2 * nwin;
    const int32_t *xwin = xoff + nd;
    const int32_t *offs = a.pat_offs + D.off_begin;
    mbar_wait(&bar, 0);
    if (!edge) {
#pragma unroll 4
        for (int d = 0; d < nd; ++d) {
            const int xo = shrink ? __ldg(xoff + d) - __ldg(xwin + d) * shrink : __ldg(xoff + d);
            const T *vd = vs + d * rc + t;
            const T *xd = xs + xo + t;
#pragma unroll
            for (int q = 0; q < Q; ++q) acc[q] = fma(vd[q * T_], xd[q * T_], acc[q]);
        }
    } else {
        for (int d = 0; d < nd; ++d) {
            const int o = __ldg(offs + d);
            const T *vd = vs + d * rc + t;
#pragma unroll
            for (int q = 0; q < Q; ++q) {
                const int64_t idx = row0 + t + q * T_ + o;
                const T xj = (idx >= a.x_lo && idx < a.x_hi) ? __ldg(a.x + idx) : T(0);
                acc[q] = fma(vd[q * T_], xj, acc[q]);
            }
        }
    }
    // scatter points in (row, col) order: gathered ones, then any beyond 32
    if (SCAT && D.nscat > 0) {
        for (unsigned m = g_mask; m; m &= m - 1) {
            const int j = __ffs(m) - 1;
            const int own = __shfl_sync(0xffffffffu, g_own, j);
            const T v = __shfl_sync(0xffffffffu, g_v, j);
            const T xv = __shfl_sync(0xffffffffu, g_x, j);
#pragma unroll
            for (int q = 0; q < Q; ++q)
                if (own == t * Q + q) acc[q] = fma(v, xv, acc[q]);
        }
        const int32_t *sr = a.scat_row + D.scat_begin;
        for (int64_t e = 32; e < D.nscat; ++e) {
            const int rr = __ldg(sr + e) - h * rc;
            if (rr < 0 || rr >= rc || rr % T_ != t) continue;
            const T v = __ldg(a.scat_val + D.scat_begin + e);
            const T xv = __ldg(a.x + __ldg(a.scat_col + D.scat_begin + e));
            const int qq = rr / T_;
#pragma unroll
            for (int j = 0; j < Q; ++j)
                if (qq == j) acc[j] = fma(v, xv, acc[j]);
        }
    }
    const T al = a.alpha, be = a.beta;
#pragma unroll
    for (int q = 0; q < Q; ++q) {
        const int64_t r = row0 + t + q * T_;
        if (!edge || r < a.nrows) {
            T *yp = a.y + r;
            const T out = (be != T(0)) ? fma(al, acc[q], be * *yp) : al * acc[q];
            __stcs(yp, out);
        }
    }
}

// ---------------------------------------------------------------------------
// Persistent, warp-specialised TMA pipeline (variant PIPE). Warp 0 (one
// elected lane) is the producer: for each segment of this CTA it stages the
// segment descriptor and the pattern's x windows into one of two x slots,
// then streams the segment's value block in chunks of up to KCH diagonals
// through a ring of NS shared-memory stages (cp.async.bulk + mbarrier
// complete_tx). The consumer warps (mrows/RPT threads) compute from shared
// memory and release stages through "empty" mbarriers. Bytes in flight are
// set by the ring depth, not by the segment size, and the descriptor and
// window fetches of the next segment overlap the current one.
// ---------------------------------------------------------------------------
constexpr int PIPE_SR = 32;  // scatter records staged per segment (one per lane)

struct PipeSeg {  // segment info handed from producer to consumers (per x slot)
    int64_t row0;
    int64_t scat_begin;
    int32_t nscat;
    int32_t flags;
    int32_t nd;
    int32_t plan_begin;
    int32_t off_begin;
    int32_t pad;
};

__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

template <typename T, int KCH, int Q>
__global__ void __launch_bounds__(544, 1) crsd_spmv_pipe(const SpmvArgs<T> a, int ns, int nx, int xmax_elems) {
    constexpr int kch = KCH;
    extern __shared__ __align__(128) unsigned char smem[];
    // layout: [bars: 2*nx + 2*ns][PipeSeg x nx][xbuf x nx][vring x ns]
    uint64_t *full_x = reinterpret_cast<uint64_t *>(smem);
    uint64_t *empty_x = full_x + nx;
    uint64_t *full_v = full_x + 2 * nx;
    uint64_t *empty_v = full_v + ns;
    PipeSeg *sseg = reinterpret_cast<PipeSeg *>(smem + ((8 * (2 * nx + 2 * ns) + 127) / 128) * 128);
    ScatRec *srec = reinterpret_cast<ScatRec *>(reinterpret_cast<unsigned char *>(sseg) + ((nx * (int)sizeof(PipeSeg) + 127) / 128) * 128);
    T *xbuf = reinterpret_cast<T *>(srec + nx * PIPE_SR);
    T *vring = xbuf + nx * (int64_t)xmax_elems;
    const int C = a.mrows / Q;  // consumer threads (Q rows each)
    const int nwarps_c = C / 32;
    const int64_t chunk_elems = (int64_t)kch * a.mrows;

    if (threadIdx.x == 0) {
        for (int i = 0; i < nx; ++i) {
            mbar_init(full_x + i, 1);
            mbar_init(empty_x + i, nwarps_c);
        }
        for (int i = 0; i < ns; ++i) {
            mbar_init(full_v + i, 1);
            mbar_init(empty_v + i, nwarps_c);
        }
        mbar_fence_init();
    }
    __syncthreads();

    if (threadIdx.x < 32) {
        // ------------------------------ producer ------------------------------
        if (threadIdx.x != 0) return;
        const uint64_t pf = policy_evict_first(), pn = policy_evict_normal();
        int xs = 0, vs = 0;
        uint32_t xph = 0, vph = 0;
        // descriptors are prefetched one segment ahead so their global-memory
        // latency overlaps the previous segment's copies
        auto seg_of = [&](int64_t w) { return a.seg_list ? (int64_t)__ldg(a.seg_list + w) : a.seg_begin + w; };
        int64_t sg_next = (blockIdx.x < a.seg_count) ? seg_of(blockIdx.x) : 0;
        SegDesc D_next;
        if (blockIdx.x < a.seg_count) D_next = a.segs[sg_next];
        for (int64_t w = blockIdx.x; w < a.seg_count; w += gridDim.x) {
            const int64_t sg = sg_next;
            const SegDesc D = D_next;
            if (w + gridDim.x < a.seg_count) {
                sg_next = seg_of(w + gridDim.x);
                D_next = a.segs[sg_next];
            }
            const int64_t row0 = sg * a.mrows;
            const bool edge = (D.flags & SEG_EDGE) != 0;
            const int32_t *plan = a.plan + D.plan_begin;
            const int nwin = __ldg(plan);
            mbar_wait(empty_x + xs, xph ^ 1);
            PipeSeg &P = sseg[xs];
            P.row0 = row0;
            P.scat_begin = D.scat_begin;
            P.nscat = D.nscat;
            P.flags = D.flags;
            P.nd = D.ndias;
            P.plan_begin = D.plan_begin;
            P.off_begin = D.off_begin;
            uint32_t xbytes = 0;
            if (!edge)
                for (int q = 0; q < nwin; ++q) xbytes += (uint32_t)__ldg(plan + 3 + 2 * q) * sizeof(T);
            const int nrec = D.nscat < PIPE_SR ? D.nscat : PIPE_SR;
            xbytes += (uint32_t)nrec * sizeof(ScatRec);
            mbar_expect_tx(full_x + xs, xbytes);  // arrive (release: P visible) + tx
            if (nrec)
                bulk_g2s(srec + xs * PIPE_SR, a.scat_rec + D.scat_begin, (uint32_t)nrec * sizeof(ScatRec), full_x + xs, pn);
            if (!edge) {
                T *dst = xbuf + (int64_t)xs * xmax_elems;
                for (int q = 0; q < nwin; ++q) {
                    const int st = __ldg(plan + 2 + 2 * q), cnt = __ldg(plan + 3 + 2 * q);
                    bulk_g2s(dst, a.x + row0 + st, (uint32_t)cnt * sizeof(T), full_x + xs, pn);
                    dst += cnt;
                }
            }
            if (++xs == nx) {
                xs = 0;
                xph ^= 1;
            }
            const int nd = D.ndias;
            for (int d0 = 0; d0 < nd; d0 += kch) {
                const int nk = min(kch, nd - d0);
                mbar_wait(empty_v + vs, vph ^ 1);
                const uint32_t bytes = (uint32_t)nk * (uint32_t)a.mrows * sizeof(T);
                mbar_expect_tx(full_v + vs, bytes);
                bulk_g2s(vring + (int64_t)vs * chunk_elems, a.vals + D.val_base + (int64_t)d0 * a.mrows, bytes,
                         full_v + vs, pf);
                if (++vs == ns) {
                    vs = 0;
                    vph ^= 1;
                }
            }
        }
        return;
    }
    // ------------------------------ consumers ------------------------------
    // Q rows per consumer thread: local rows ct + q*C (conflict-free shared reads)
    const int ct = threadIdx.x - 32;
    const int lane = ct & 31;
    int xs = 0, vs = 0;
    uint32_t xph = 0, vph = 0;
    const T al = a.alpha, be = a.beta;
    for (int64_t w = blockIdx.x; w < a.seg_count; w += gridDim.x) {
        mbar_wait(full_x + xs, xph);
        const PipeSeg P = sseg[xs];
        const bool edge = (P.flags & SEG_EDGE) != 0;
        const int32_t *plan = a.plan + P.plan_begin;
        const int nwin = __ldg(plan);
        const int32_t *xoff = plan + 2 + 2 * nwin;
        const int32_t *offs = a.pat_offs + P.off_begin;
        const T *xb = xbuf + (int64_t)xs * xmax_elems + ct;
        // scatter points: each warp gathers the entries owned by its threads
        // now (lane l takes entry l of the first 32 of the segment; a ballot
        // keeps the ones whose row belongs to this warp), so the random x
        // loads are in flight during the diagonal loop; entries beyond 32 are
        // read at the end (rare)
        int g_own = -1;
        T g_v = T(0), g_x = T(0);
        unsigned g_mask = 0u;
        if (P.nscat > 0) {
            // the first PIPE_SR points arrived with the slot as 32-B records:
            // only the x[col] gather is a global load, issued now
            const ScatRec *R = srec + xs * PIPE_SR;
            if (lane < P.nscat) {
                const int rr = R[lane].row;
                g_own = (rr % C) * Q + rr / C;  // (thread, slot)
            }
            const bool mine = g_own >= 0 && (g_own / Q) / 32 == ct / 32;
            g_mask = __ballot_sync(0xffffffffu, mine);
            if (mine) {
                g_v = *reinterpret_cast<const T *>(&R[lane].val);
                g_x = __ldg(a.x + R[lane].col);
            }
        }
        T acc[Q];
#pragma unroll
        for (int q = 0; q < Q; ++q) acc[q] = T(0);
        for (int d0 = 0; d0 < P.nd; d0 += kch) {
            const int nk = min(kch, P.nd - d0);
            mbar_wait(full_v + vs, vph);
            const T *vb = vring + (int64_t)vs * chunk_elems + ct;
            if (!edge) {
                int xo[KCH];
#pragma unroll
                for (int k = 0; k < KCH; ++k)
                    if (k < nk) xo[k] = __ldg(xoff + d0 + k);
#pragma unroll
                for (int k = 0; k < KCH; ++k)
                    if (k < nk) {
#pragma unroll
                        for (int q = 0; q < Q; ++q) acc[q] = fma(vb[k * a.mrows + q * C], xb[xo[k] + q * C], acc[q]);
                    }
            } else {
                for (int k = 0; k < nk; ++k) {
                    const int o = __ldg(offs + d0 + k);
#pragma unroll
                    for (int q = 0; q < Q; ++q) {
                        const int64_t idx = P.row0 + ct + q * C + o;
                        const T xj = (idx >= a.x_lo && idx < a.x_hi) ? __ldg(a.x + idx) : T(0);
                        acc[q] = fma(vb[k * a.mrows + q * C], xj, acc[q]);
                    }
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(empty_v + vs);
            if (++vs == ns) {
                vs = 0;
                vph ^= 1;
            }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(empty_x + xs);  // the x slot is no longer needed
        // scatter points in (row, col) order: the gathered ones (broadcast
        // from the lane that holds them), then any beyond 32
        if (P.nscat > 0) {
            for (unsigned m = g_mask; m; m &= m - 1) {
                const int j = __ffs(m) - 1;
                const int own = __shfl_sync(0xffffffffu, g_own, j);
                const T v = __shfl_sync(0xffffffffu, g_v, j);
                const T xv = __shfl_sync(0xffffffffu, g_x, j);
#pragma unroll
                for (int q = 0; q < Q; ++q)
                    if (own == ct * Q + q) acc[q] = fma(v, xv, acc[q]);
            }
            const int32_t *sr = a.scat_row + P.scat_begin;
            for (int64_t e = 32; e < P.nscat; ++e) {
                const int rr = __ldg(sr + e);
                if (rr % C != ct) continue;
                const T v = __ldg(a.scat_val + P.scat_begin + e);
                const T xv = __ldg(a.x + __ldg(a.scat_col + P.scat_begin + e));
                const int qq = rr / C;
#pragma unroll
                for (int q = 0; q < Q; ++q)
                    if (qq == q) acc[q] = fma(v, xv, acc[q]);
            }
        }
#pragma unroll
        for (int q = 0; q < Q; ++q) {
            const int64_t row = P.row0 + ct + q * C;
            if (!edge || row < a.nrows) {
                T *yp = a.y + row;
                __stcs(yp, (be != T(0)) ? fma(al, acc[q], be * *yp) : al * acc[q]);
            }
        }
        if (++xs == nx) {
            xs = 0;
            xph ^= 1;
        }
    }
}

// shared memory of the PIPE variant for nx x slots and ns value stages
inline int64_t pipe_smem(int ns, int nx, int kch, int mrows, int elem, int64_t xmax_elems) {
    const int64_t bars = ((8 * (2 * nx + 2 * ns) + 127) / 128) * 128;
    const int64_t segs = ((nx * (int64_t)sizeof(PipeSeg) + 127) / 128) * 128;
    const int64_t recs = nx * PIPE_SR * (int64_t)sizeof(ScatRec);
    return bars + segs + recs + nx * xmax_elems * elem + (int64_t)ns * kch * mrows * elem;
}

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) applies per device
// context: remember the largest size set, per device and kernel instance.
constexpr int kMaxDev = 64;
static std::mutex g_attr_mu;
template <typename K>
static cudaError_t ensure_smem(K kern, int bytes, int *cache_per_dev) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= kMaxDev) return cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    std::lock_guard<std::mutex> lk(g_attr_mu);
    if (bytes <= cache_per_dev[dev]) return cudaSuccess;
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess) cache_per_dev[dev] = bytes;
    return e;
}

template <typename T>
int launch_spmv(const SpmvArgs<T> &a, int sm_count, void *stream) {
    if (a.seg_count <= 0) return 0;
    constexpr int R = VecT<T>::R;
    const int threads = a.mrows / R;
    int64_t grid = a.seg_count;
    if (grid > 0x7fffffff) grid = 0x7fffffff;
    cudaError_t e;
    if (a.variant == VARIANT_TMA) {
        const int split = a.tma_split, q = a.tma_q;
        const int rc = a.mrows / split;
        const int thr = rc / q;
        const int smem = (int)a.tma_smem;
        static int attr_bytes[3][2][kMaxDev] = {};
        const int qi = q == 1 ? 0 : (q == 2 ? 1 : 2);
        const bool sc = a.has_scatter != 0;
        auto kern = sc ? (q == 1 ? crsd_spmv_tma<T, 1, true> : (q == 2 ? crsd_spmv_tma<T, 2, true> : crsd_spmv_tma<T, 4, true>))
                       : (q == 1 ? crsd_spmv_tma<T, 1, false> : (q == 2 ? crsd_spmv_tma<T, 2, false> : crsd_spmv_tma<T, 4, false>));
        e = ensure_smem(kern, smem, attr_bytes[qi][sc]);
        if (e != cudaSuccess) return -(10000 + (int)e);
        int64_t g = a.seg_count * split;
        if (g > 0x7fffffff) g = 0x7fffffff;
        kern<<<(unsigned)g, thr, smem, (cudaStream_t)stream>>>(a, split);
    } else if (a.variant == VARIANT_PIPE) {
        // ring of KCH-diagonal value chunks; Q rows per consumer thread so a
        // CTA has <= 256 consumers; two CTAs per SM, nx x slots, as many
        // stages as fit
        constexpr int kch = 8;
        const int64_t xmax = a.pipe_xmax_elems;
        const int q = a.mrows > 256 ? a.mrows / 256 : 1;
        const int C = a.mrows / q;
        const int per_sm = C <= 256 ? 2 : 1;
        const int64_t budget = (per_sm >= 2 ? 110 : 220) * 1024;
        const int nx = 2;
        int ns = 32;
        while (ns > 2 && pipe_smem(ns, nx, kch, a.mrows, sizeof(T), xmax) > budget) --ns;
        const int64_t sm = pipe_smem(ns, nx, kch, a.mrows, sizeof(T), xmax);
        static int attr_pipe[3][kMaxDev] = {};
        const int qi = q == 1 ? 0 : (q == 2 ? 1 : 2);
        auto kern = q == 1 ? crsd_spmv_pipe<T, kch, 1> : (q == 2 ? crsd_spmv_pipe<T, kch, 2> : crsd_spmv_pipe<T, kch, 4>);
        e = ensure_smem(kern, (int)sm, attr_pipe[qi]);
        if (e != cudaSuccess) return -(10000 + (int)e);
        int64_t g = (int64_t)sm_count * per_sm;
        if (g > a.seg_count) g = a.seg_count;
        kern<<<(unsigned)g, C + 32, sm, (cudaStream_t)stream>>>(a, ns, nx, (int)xmax);
    } else {
        crsd_spmv_ldg<T, 4><<<(unsigned)grid, threads, 0, (cudaStream_t)stream>>>(a);
    }
    e = cudaGetLastError();
    return e == cudaSuccess ? 1 : -(int)e;
}

// ---------------------------------------------------------------------------
// Paper-exact scatter rows (CRSD_PAPER_ELL; P:L395-411 storage, P:L703-719
// "the final kernel is composed of two parts": the ELL part runs after the
// diagonal part and overwrites y for the rows it stores). One thread per
// stored row, column-major ELL (coalesced across threads), the row product
// accumulated in ascending column order with separately rounded multiply and
// add -- the CSR evaluation order, reproducible bit for bit.
// ---------------------------------------------------------------------------
__device__ __forceinline__ double mul_rn(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ float mul_rn(float a, float b) { return __fmul_rn(a, b); }
__device__ __forceinline__ double add_rn(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ float add_rn(float a, float b) { return __fadd_rn(a, b); }

template <typename T>
__global__ void __launch_bounds__(256) crsd_paper_ell(const int64_t *__restrict__ rowno, const int64_t *__restrict__ col,
                                                      const T *__restrict__ val, int64_t n, int64_t width,
                                                      const T *__restrict__ x, T *__restrict__ y, T alpha) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    T s = T(0);
    for (int64_t k = 0; k < width; ++k) {
        const int64_t c = __ldg(col + k * n + i);
        if (c < 0) break;  // rows are left-packed: padding only at the end
        s = add_rn(s, mul_rn(__ldg(val + k * n + i), __ldg(x + c)));
    }
    y[__ldg(rowno + i)] = mul_rn(alpha, s);
}

template <typename T>
int launch_paper_ell(const int64_t *rowno, const int64_t *col, const T *val, int64_t n, int64_t width, const T *x,
                     T *y, T alpha, void *stream) {
    if (n <= 0) return 0;
    crsd_paper_ell<T><<<(unsigned)((n + 255) / 256), 256, 0, (cudaStream_t)stream>>>(rowno, col, val, n, width, x, y, alpha);
    return (int)cudaGetLastError();
}

template int launch_paper_ell<double>(const int64_t *, const int64_t *, const double *, int64_t, int64_t,
                                      const double *, double *, double, void *);
template int launch_paper_ell<float>(const int64_t *, const int64_t *, const float *, int64_t, int64_t, const float *,
                                     float *, float, void *);

template int launch_spmv<double>(const SpmvArgs<double> &, int, void *);
template int launch_spmv<float>(const SpmvArgs<float> &, int, void *);

}  // namespace crsd
