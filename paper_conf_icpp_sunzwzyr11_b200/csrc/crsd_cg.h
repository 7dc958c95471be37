// Device state and kernel launchers of the CG iteration (cg.cu, solver.cpp).
#pragma once

#include <cstdint>

namespace crsd {

enum { CG_PQ = 0, CG_RR = 1, CG_BB = 2 };  // reduction slots (red[RR], red[BB] adjacent: one allreduce)

// Scalars of the iteration, resident in device memory for the whole solve.
struct CgState {
    double red[4];       // reduction slots: rank-local sums, then (multi-GPU) allreduced in place
    double rr;           // (r_j, r_j) of the current step (global)
    double bb;           // (b, b)
    double rtol;         // stopping test sqrt(rr) <= rtol * sqrt(bb)
    double tol2;         // rtol^2 * bb
    int64_t it;          // steps taken
    int64_t max_iter;
    int64_t hist_cap;    // hist has hist_cap + 1 entries
    double *hist;        // (r_j, r_j) for j = 0..it, or null
    double *partials;    // one per CTA of the vector kernels
    uint32_t counter;    // last-CTA detection (reset by the last CTA)
    int32_t done;        // stopping test met or max_iter reached: the vector kernels become no-ops
};

int cg_grid(int sm_count);
template <typename T>
int cg_launch_dot(const T *a, const T *b, int64_t n, CgState *st, int slot, bool skip_if_done, int grid, void *stream);
template <typename T>
int cg_launch_update(T *r, const T *q, int64_t n, CgState *st, int grid, void *stream);
template <typename T>
int cg_launch_pupdate(T *p, const T *r, T *x, int64_t n, CgState *st, int grid, void *stream);
int cg_launch_init(CgState *st, void *stream);

}  // namespace crsd
