// Vector kernels of the conjugate gradient iteration built on the CRSD SpMV
// (the FDM/FVM PDE use case the paper motivates CRSD
// with; textbook CG, Hestenes & Stiefel / Saad Alg. 6.18, the
// paper's reference [2]).
//
// Per step j (crsd_cg in solver.cpp):
//   q = A p                      CRSD SpMV (any variant)
//   (p, q)                       cg_dot         -> red[PQ]   [NCCL allreduce]
//   alpha = rr / (p, q)
//   r -= alpha q, (r, r)         cg_update      -> red[RR]   [NCCL allreduce]
//   beta = (r,r)_new / rr        cg_pupdate     -> rr, it, done
//   x += alpha p, p = r + beta p
// All scalars live on the device (CgState), so a batch of steps is one CUDA
// graph with no host round trip; the stopping test is taken on the device
// after every step (the host only polls `done` between batches). Dot products
// accumulate in fp64 for both matrix precisions and reduce deterministically:
// per-CTA partials, summed in CTA order by the last CTA to finish.
//
// These kernels are HBM-bound streams (no reuse): grid = resident CTAs of
// the whole GPU, 128-bit loads and stores, grid-stride loop.
#include <cuda_runtime.h>

#include <cstdint>

#include "crsd_cg.h"

namespace crsd {

namespace {

constexpr int CG_THREADS = 512;

template <typename T>
struct Vec;
template <>
struct Vec<double> {
    using type = double2;
    static constexpr int R = 2;
};
template <>
struct Vec<float> {
    using type = float4;
    static constexpr int R = 4;
};

__device__ __forceinline__ double el(const double2 &v, int j) { return j == 0 ? v.x : v.y; }
__device__ __forceinline__ float el(const float4 &v, int j) {
    return j == 0 ? v.x : (j == 1 ? v.y : (j == 2 ? v.z : v.w));
}
__device__ __forceinline__ void set(double2 &v, int j, double s) {
    if (j == 0) v.x = s; else v.y = s;
}
__device__ __forceinline__ void set(float4 &v, int j, float s) {
    if (j == 0) v.x = s; else if (j == 1) v.y = s; else if (j == 2) v.z = s; else v.w = s;
}

__device__ __forceinline__ double block_sum(double v) {
    __shared__ double ws[CG_THREADS / 32];
    for (int o = 16; o; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    __syncthreads();  // ws may still be read by a previous call
    if (l == 0) ws[w] = v;
    __syncthreads();
    v = 0.0;
    if (w == 0) {
        v = l < (int)(blockDim.x >> 5) ? ws[l] : 0.0;
        for (int o = 16; o; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
    }
    return v;  // valid in thread 0
}

// Deterministic grid reduction: every CTA stores its partial, the last CTA to
// arrive sums the partials in CTA order. Returns true in thread 0 of the last
// CTA, with the total in `total`.
__device__ __forceinline__ bool grid_sum(double v, double *partials, uint32_t *counter, double &total) {
    __shared__ bool last;
    v = block_sum(v);
    if (threadIdx.x == 0) {
        partials[blockIdx.x] = v;
        __threadfence();
        last = atomicAdd(counter, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!last) return false;
    __threadfence();
    double s = 0.0;
    for (int i = threadIdx.x; i < (int)gridDim.x; i += blockDim.x) s += *((volatile double *)partials + i);
    s = block_sum(s);
    if (threadIdx.x == 0) {
        total = s;
        *counter = 0u;
        return true;
    }
    return false;
}

// Completion counter for kernels without a reduction: true in thread 0 of the
// last CTA (after every CTA has read the state it needs).
__device__ __forceinline__ bool grid_last(uint32_t *counter) {
    __shared__ bool last;
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        last = atomicAdd(counter, 1u) == gridDim.x - 1;
        if (last) *counter = 0u;
    }
    __syncthreads();
    return threadIdx.x == 0 && last;
}

template <typename T>
__global__ void __launch_bounds__(CG_THREADS) cg_dot(const T *__restrict__ a, const T *__restrict__ b, int64_t n,
                                                     CgState *st, int slot, int skip_if_done) {
    if (skip_if_done && *(volatile int32_t *)&st->done) return;
    using V = typename Vec<T>::type;
    constexpr int R = Vec<T>::R;
    const int64_t nv = n / R;
    const V *av = reinterpret_cast<const V *>(a), *bv = reinterpret_cast<const V *>(b);
    double s = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nv; i += (int64_t)gridDim.x * blockDim.x) {
        const V u = __ldcs(av + i), w = __ldcs(bv + i);
#pragma unroll
        for (int j = 0; j < R; ++j) s = fma((double)el(u, j), (double)el(w, j), s);
    }
    if (blockIdx.x == 0)
        for (int64_t i = nv * R + threadIdx.x; i < n; i += blockDim.x) s = fma((double)a[i], (double)b[i], s);
    double tot;
    if (grid_sum(s, st->partials, &st->counter, tot)) st->red[slot] = tot;
}

// r -= alpha q; red[RR] = (r, r)   (alpha = rr / (p, q))
template <typename T>
__global__ void __launch_bounds__(CG_THREADS) cg_update(T *__restrict__ r, const T *__restrict__ q, int64_t n,
                                                        CgState *st) {
    if (*(volatile int32_t *)&st->done) return;
    using V = typename Vec<T>::type;
    constexpr int R = Vec<T>::R;
    const T alpha = (T)(st->rr / st->red[CG_PQ]);
    const int64_t nv = n / R;
    V *rv = reinterpret_cast<V *>(r);
    const V *qv = reinterpret_cast<const V *>(q);
    double s = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nv; i += (int64_t)gridDim.x * blockDim.x) {
        V rr = __ldcs(rv + i);
        const V qq = __ldcs(qv + i);
#pragma unroll
        for (int j = 0; j < R; ++j) {
            const T rn = fma(-alpha, el(qq, j), el(rr, j));
            set(rr, j, rn);
            s = fma((double)rn, (double)rn, s);
        }
        __stcs(rv + i, rr);
    }
    if (blockIdx.x == 0)
        for (int64_t i = nv * R + threadIdx.x; i < n; i += blockDim.x) {
            const T rn = fma(-alpha, q[i], r[i]);
            r[i] = rn;
            s = fma((double)rn, (double)rn, s);
        }
    double tot;
    if (grid_sum(s, st->partials, &st->counter, tot)) st->red[CG_RR] = tot;
}

// x += alpha p (with the p of this step), then p = r + beta p
// (beta = red[RR] / rr); the last CTA advances the state: rr = red[RR],
// it += 1, history, stopping test. Moving the x update here (it needs only
// alpha and the old p) saves one read of p and one pass over x.
template <typename T>
__global__ void __launch_bounds__(CG_THREADS) cg_pupdate(T *__restrict__ p, const T *__restrict__ r,
                                                         T *__restrict__ x, int64_t n, CgState *st) {
    if (*(volatile int32_t *)&st->done) return;
    using V = typename Vec<T>::type;
    constexpr int R = Vec<T>::R;
    const double rr_new = st->red[CG_RR];
    const T alpha = (T)(st->rr / st->red[CG_PQ]);
    const T beta = (T)(rr_new / st->rr);
    const int64_t nv = n / R;
    V *pv = reinterpret_cast<V *>(p), *xv = reinterpret_cast<V *>(x);
    const V *rv = reinterpret_cast<const V *>(r);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nv; i += (int64_t)gridDim.x * blockDim.x) {
        V pp = __ldcs(pv + i), xx = __ldcs(xv + i);
        const V rr = __ldcs(rv + i);
#pragma unroll
        for (int j = 0; j < R; ++j) {
            set(xx, j, fma(alpha, el(pp, j), el(xx, j)));
            set(pp, j, fma(beta, el(pp, j), el(rr, j)));
        }
        __stcs(xv + i, xx);
        __stcs(pv + i, pp);
    }
    if (blockIdx.x == 0)
        for (int64_t i = nv * R + threadIdx.x; i < n; i += blockDim.x) {
            x[i] = fma(alpha, p[i], x[i]);
            p[i] = fma(beta, p[i], r[i]);
        }
    if (grid_last(&st->counter)) {
        st->rr = rr_new;
        st->it += 1;
        if (st->hist && st->it <= st->hist_cap) st->hist[st->it] = rr_new;
        st->done = (rr_new <= st->tol2 || st->it >= st->max_iter) ? 1 : 0;
    }
}

__global__ void cg_init(CgState *st) {
    st->rr = st->red[CG_RR];
    st->bb = st->red[CG_BB];
    st->tol2 = st->rtol * st->rtol * st->bb;
    st->it = 0;
    if (st->hist) st->hist[0] = st->rr;
    st->done = (st->rr <= st->tol2 || st->max_iter <= 0) ? 1 : 0;
}

}  // namespace

int cg_grid(int sm_count) { return sm_count * (2048 / CG_THREADS); }

template <typename T>
int cg_launch_dot(const T *a, const T *b, int64_t n, CgState *st, int slot, bool skip_if_done, int grid, void *stream) {
    cg_dot<T><<<grid, CG_THREADS, 0, (cudaStream_t)stream>>>(a, b, n, st, slot, skip_if_done ? 1 : 0);
    return (int)cudaGetLastError();
}
template <typename T>
int cg_launch_update(T *r, const T *q, int64_t n, CgState *st, int grid, void *stream) {
    cg_update<T><<<grid, CG_THREADS, 0, (cudaStream_t)stream>>>(r, q, n, st);
    return (int)cudaGetLastError();
}
template <typename T>
int cg_launch_pupdate(T *p, const T *r, T *x, int64_t n, CgState *st, int grid, void *stream) {
    cg_pupdate<T><<<grid, CG_THREADS, 0, (cudaStream_t)stream>>>(p, r, x, n, st);
    return (int)cudaGetLastError();
}
int cg_launch_init(CgState *st, void *stream) {
    cg_init<<<1, 1, 0, (cudaStream_t)stream>>>(st);
    return (int)cudaGetLastError();
}

template int cg_launch_dot<double>(const double *, const double *, int64_t, CgState *, int, bool, int, void *);
template int cg_launch_dot<float>(const float *, const float *, int64_t, CgState *, int, bool, int, void *);
template int cg_launch_update<double>(double *, const double *, int64_t, CgState *, int, void *);
template int cg_launch_update<float>(float *, const float *, int64_t, CgState *, int, void *);
template int cg_launch_pupdate<double>(double *, const double *, double *, int64_t, CgState *, int, void *);
template int cg_launch_pupdate<float>(float *, const float *, float *, int64_t, CgState *, int, void *);

}  // namespace crsd
