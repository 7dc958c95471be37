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

constexpr int SCAT_STAGE = 128;

// A CTA covers `rc` rows of one segment (rc = mrows / split): with split > 1
// the segment's value block is fetched as one bulk copy per diagonal (its rc
// consecutive values), so big segments (many diagonals) still leave several
// CTAs resident per SM. Thread t owns rows t + q*(rc/Q), q < Q.
template <typename T, int Q>
__global__ void __launch_bounds__(256) crsd_spmv_tma(const SpmvArgs<T> a, int split) {
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t bar;
    const int t = threadIdx.x;
    const int T_ = blockDim.x;
    const int rc = a.mrows / split;  // rows of this CTA
    const int64_t cta = a.seg_list ? (int64_t)blockIdx.x : (int64_t)blockIdx.x;
    const int64_t w = cta / split;
    const int h = (int)(cta - w * split);
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
        // warp 0 issues the remaining copies, window / diagonal q by lane q % 32
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
    // Scatter points of this CTA's rows are gathered now, while the bulk
    // copies are in flight: thread e loads entry e (value, x[col], owner), so
    // the random x reads overlap the TMA wait instead of ending the CTA.
    __shared__ T sc_v[SCAT_STAGE], sc_x[SCAT_STAGE];
    __shared__ int32_t sc_own[SCAT_STAGE];
    const int nst = D.nscat < SCAT_STAGE ? D.nscat : SCAT_STAGE;
    if (t < nst) {
        const int rr = __ldg(a.scat_row + D.scat_begin + t) - h * rc;
        int own = -1;
        if (rr >= 0 && rr < rc) own = (rr % T_) * Q + rr / T_;  // (thread, slot)
        sc_own[t] = own;
        if (own >= 0) {
            sc_v[t] = __ldg(a.scat_val + D.scat_begin + t);
            sc_x[t] = __ldg(a.x + __ldg(a.scat_col + D.scat_begin + t));
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
    // scatter points in (row, col) order: staged ones from shared memory,
    // any beyond SCAT_STAGE from global memory
    if (D.nscat > 0) {
        __syncthreads();
        for (int e = 0; e < nst; ++e) {
            const int own = sc_own[e];
            if (own < 0 || own / Q != t) continue;
#pragma unroll
            for (int j = 0; j < Q; ++j)
                if (own - t * Q == j) acc[j] = fma(sc_v[e], sc_x[e], acc[j]);
        }
        const int32_t *sr = a.scat_row + D.scat_begin;
        for (int64_t e = nst; e < D.nscat; ++e) {
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
// Persistent, double-buffered TMA variant (PIPE). Each CTA walks work items
// i = blockIdx.x, +gridDim.x, ... (item = one row slice of one segment, as in
// crsd_spmv_tma) with two shared-memory slots: while it computes item i from
// one slot, the bulk copies of item i + G are already landing in the other,
// and thread 0 has the descriptor of the item after that in registers. The
// scatter points of the next item are gathered (value, x[col]) into a
// double-buffered staging area while the current item computes. This keeps
// segment-descriptor latency and scatter gathers off the critical path that
// bounds the one-shot variant (CTA launch -> descriptor -> copies -> wait).
// ---------------------------------------------------------------------------
struct SlotInfo {
    int64_t row0;
    int64_t scat_begin;
    int32_t nscat, flags, nd, plan_begin, off_begin, h;
};

__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

template <typename T, int Q>
__global__ void __launch_bounds__(256) crsd_spmv_tmap(const SpmvArgs<T> a, int split, int slot_elems) {
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t bar[2];
    __shared__ SlotInfo info[2];
    __shared__ T sc_v[2][SCAT_STAGE], sc_x[2][SCAT_STAGE];
    __shared__ int32_t sc_own[2][SCAT_STAGE];
    const int t = threadIdx.x;
    const int T_ = blockDim.x;
    const int rc = a.mrows / split;
    const int shrink = a.mrows - rc;
    const int64_t nitems = a.seg_count * split;
    const int64_t G = gridDim.x;
    T *slot0 = reinterpret_cast<T *>(smem);

    auto seg_of = [&](int64_t item, int &h) {
        const int64_t w = item / split;
        h = (int)(item - w * split);
        return a.seg_list ? (int64_t)__ldg(a.seg_list + w) : a.seg_begin + w;
    };
    // thread 0: publish item info in slot sl and issue its bulk copies
    auto issue = [&](int sl, int64_t sg, int h, const SegDesc &D) {
        SlotInfo &I = info[sl];
        I.row0 = sg * a.mrows + (int64_t)h * rc;
        I.scat_begin = D.scat_begin;
        I.nscat = D.nscat;
        I.flags = D.flags;
        I.nd = D.ndias;
        I.plan_begin = D.plan_begin;
        I.off_begin = D.off_begin;
        I.h = h;
        const int32_t *plan = a.plan + D.plan_begin;
        const int nwin = __ldg(plan);
        const bool edge = (D.flags & SEG_EDGE) != 0;
        const int nd = D.ndias;
        const uint32_t vbytes = (uint32_t)nd * (uint32_t)rc * sizeof(T);
        const uint32_t xfull = (uint32_t)__ldg(plan + 1) - (uint32_t)nd * (uint32_t)a.mrows * sizeof(T);
        const uint32_t xbytes = edge ? 0u : xfull - (uint32_t)(nwin * shrink) * sizeof(T);
        T *vs = slot0 + (int64_t)sl * slot_elems;
        T *xs = vs + (int64_t)nd * rc;
        mbar_expect_tx(bar + sl, vbytes + xbytes);  // arrive (release: info visible)
        const uint64_t pf = policy_evict_first();
        if (split == 1) {
            if (vbytes) bulk_g2s(vs, a.vals + D.val_base, vbytes, bar + sl, pf);
        } else {
            for (int d = 0; d < nd; ++d)
                bulk_g2s(vs + (int64_t)d * rc, a.vals + D.val_base + (int64_t)d * a.mrows + (int64_t)h * rc,
                         (uint32_t)rc * sizeof(T), bar + sl, pf);
        }
        if (!edge) {
            const uint64_t pn = policy_evict_normal();
            T *dst = xs;
            for (int q = 0; q < nwin; ++q) {
                const int st = __ldg(plan + 2 + 2 * q), cnt = __ldg(plan + 3 + 2 * q) - shrink;
                bulk_g2s(dst, a.x + I.row0 + st, (uint32_t)cnt * sizeof(T), bar + sl, pn);
                dst += cnt;
            }
        }
    };
    // all threads: gather the scatter points of the item in slot sl
    auto gather = [&](int sl) {
        const SlotInfo &I = info[sl];
        const int nst = I.nscat < SCAT_STAGE ? I.nscat : SCAT_STAGE;
        for (int e = t; e < nst; e += T_) {
            const int rr = __ldg(a.scat_row + I.scat_begin + e) - I.h * rc;
            int own = -1;
            if (rr >= 0 && rr < rc) own = (rr % T_) * Q + rr / T_;
            sc_own[sl][e] = own;
            if (own >= 0) {
                sc_v[sl][e] = __ldg(a.scat_val + I.scat_begin + e);
                sc_x[sl][e] = __ldg(a.x + __ldg(a.scat_col + I.scat_begin + e));
            }
        }
    };

    SegDesc Dn;
    int64_t sn = 0;
    int hn = 0;
    if (t == 0) {
        mbar_init(bar, 1);
        mbar_init(bar + 1, 1);
        mbar_fence_init();
        int h;
        for (int k = 0; k < 2; ++k) {
            const int64_t it = blockIdx.x + k * G;
            if (it < nitems) {
                const int64_t sg = seg_of(it, h);
                const SegDesc D = a.segs[sg];
                issue(k, sg, h, D);
            }
        }
        if (blockIdx.x + 2 * G < nitems) {
            sn = seg_of(blockIdx.x + 2 * G, hn);
            Dn = a.segs[sn];
        }
    }
    __syncthreads();
    if (blockIdx.x < nitems) gather(0);
    __syncthreads();

    const T al = a.alpha, be = a.beta;
    uint32_t ph0 = 0, ph1 = 0;
    int k = 0;
    for (int64_t it = blockIdx.x; it < nitems; it += G, ++k) {
        const int sl = k & 1;
        if (it + G < nitems) gather(sl ^ 1);  // next item's scatter points
        mbar_wait(bar + sl, sl ? ph1 : ph0);
        if (sl) ph1 ^= 1; else ph0 ^= 1;
        const SlotInfo I = info[sl];
        const bool edge = (I.flags & SEG_EDGE) != 0;
        const int32_t *plan = a.plan + I.plan_begin;
        const int nwin = __ldg(plan);
        const int32_t *xoff = plan + 2 + 2 * nwin;
        const int32_t *xwin = xoff + I.nd;
        const int32_t *offs = a.pat_offs + I.off_begin;
        const T *vs = slot0 + (int64_t)sl * slot_elems;
        const T *xs = vs + (int64_t)I.nd * rc;
        T acc[Q];
#pragma unroll
        for (int q = 0; q < Q; ++q) acc[q] = T(0);
        if (!edge) {
#pragma unroll 4
            for (int d = 0; d < I.nd; ++d) {
                const int xo = shrink ? __ldg(xoff + d) - __ldg(xwin + d) * shrink : __ldg(xoff + d);
                const T *vd = vs + d * rc + t;
                const T *xd = xs + xo + t;
#pragma unroll
                for (int q = 0; q < Q; ++q) acc[q] = fma(vd[q * T_], xd[q * T_], acc[q]);
            }
        } else {
            for (int d = 0; d < I.nd; ++d) {
                const int o = __ldg(offs + d);
                const T *vd = vs + d * rc + t;
#pragma unroll
                for (int q = 0; q < Q; ++q) {
                    const int64_t idx = I.row0 + t + q * T_ + o;
                    const T xj = (idx >= a.x_lo && idx < a.x_hi) ? __ldg(a.x + idx) : T(0);
                    acc[q] = fma(vd[q * T_], xj, acc[q]);
                }
            }
        }
        if (I.nscat > 0) {
            const int nst = I.nscat < SCAT_STAGE ? I.nscat : SCAT_STAGE;
            for (int e = 0; e < nst; ++e) {
                const int own = sc_own[sl][e];
                if (own < 0 || own / Q != t) continue;
#pragma unroll
                for (int j = 0; j < Q; ++j)
                    if (own - t * Q == j) acc[j] = fma(sc_v[sl][e], sc_x[sl][e], acc[j]);
            }
            for (int64_t e = nst; e < I.nscat; ++e) {
                const int rr = __ldg(a.scat_row + I.scat_begin + e) - I.h * rc;
                if (rr < 0 || rr >= rc || rr % T_ != t) continue;
                const T v = __ldg(a.scat_val + I.scat_begin + e);
                const T xv = __ldg(a.x + __ldg(a.scat_col + I.scat_begin + e));
                const int qq = rr / T_;
#pragma unroll
                for (int j = 0; j < Q; ++j)
                    if (qq == j) acc[j] = fma(v, xv, acc[j]);
            }
        }
#pragma unroll
        for (int q = 0; q < Q; ++q) {
            const int64_t r = I.row0 + t + q * T_;
            if (!edge || r < a.nrows) {
                T *yp = a.y + r;
                __stcs(yp, (be != T(0)) ? fma(al, acc[q], be * *yp) : al * acc[q]);
            }
        }
        __syncthreads();  // slot sl, info[sl], staging[sl] free; staging[sl^1] written
        if (t == 0 && it + 2 * G < nitems) {
            fence_proxy_async_smem();
            issue(sl, sn, hn, Dn);
            if (it + 3 * G < nitems) {
                sn = seg_of(it + 3 * G, hn);
                Dn = a.segs[sn];
            }
        }
        __syncthreads();  // info[sl] of item it + 2G visible for the next gather
    }
}

static int env_int(const char *k, int d) {
    const char *v = getenv(k);
    return v ? atoi(v) : d;
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
        static int attr_bytes[2][3] = {{0, 0, 0}, {0, 0, 0}};
        const int qi = q == 1 ? 0 : (q == 2 ? 1 : 2);
        int &cur = attr_bytes[sizeof(T) == 8][qi];
        auto kern = q == 1 ? crsd_spmv_tma<T, 1> : (q == 2 ? crsd_spmv_tma<T, 2> : crsd_spmv_tma<T, 4>);
        if (smem > cur) {
            e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e != cudaSuccess) return -(10000 + (int)e);
            cur = smem;
        }
        int64_t g = a.seg_count * split;
        if (g > 0x7fffffff) g = 0x7fffffff;
        kern<<<(unsigned)g, thr, smem, (cudaStream_t)stream>>>(a, split);
    } else if (a.variant == VARIANT_PIPE) {
        const int split = a.tma_split, q = a.tma_q;
        const int rc = a.mrows / split;
        const int thr = rc / q;
        const int slot_elems = (int)((a.tma_smem / sizeof(T) + 31) / 32 * 32);
        const int smem = 2 * slot_elems * (int)sizeof(T);
        static int attr_p[2][3] = {{0, 0, 0}, {0, 0, 0}};
        const int qi = q == 1 ? 0 : (q == 2 ? 1 : 2);
        int &cur = attr_p[sizeof(T) == 8][qi];
        auto kern = q == 1 ? crsd_spmv_tmap<T, 1> : (q == 2 ? crsd_spmv_tmap<T, 2> : crsd_spmv_tmap<T, 4>);
        if (smem > cur) {
            e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e != cudaSuccess) return -(10000 + (int)e);
            cur = smem;
        }
        int per_sm = 0;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, thr, smem);
        if (e != cudaSuccess || per_sm < 1) per_sm = 1;
        per_sm = env_int("CRSD_PIPE_PERSM", per_sm);
        int64_t g = (int64_t)sm_count * per_sm;
        const int64_t nitems = a.seg_count * split;
        if (g > nitems) g = nitems;
        kern<<<(unsigned)g, thr, smem, (cudaStream_t)stream>>>(a, split, slot_elems);
    } else {
        crsd_spmv_ldg<T, 4><<<(unsigned)grid, threads, 0, (cudaStream_t)stream>>>(a);
    }
    e = cudaGetLastError();
    return e == cudaSuccess ? 1 : -(int)e;
}

template int launch_spmv<double>(const SpmvArgs<double> &, int, void *);
template int launch_spmv<float>(const SpmvArgs<float> &, int, void *);

}  // namespace crsd
