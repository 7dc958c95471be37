"""ORACLE (test infrastructure only; the product never imports it): the
conjugate gradient method for a symmetric positive definite A, written out in
the textbook order (Hestenes & Stiefel 1952; Saad, "Iterative Methods for
Sparse Linear Systems", Algorithm 6.18 -- reference [2] of the paper,
PAPER.md P:L1367). The paper motivates CRSD with the coefficient matrices of
FDM/FVM discretisations of PDEs, whose solution is the iteration
below with one SpMV per step.

    r_0 = b - A x_0,  p_0 = r_0
    for j = 0, 1, ...:
        q_j       = A p_j
        alpha_j   = (r_j, r_j) / (p_j, q_j)
        x_{j+1}   = x_j + alpha_j p_j
        r_{j+1}   = r_j - alpha_j q_j
        beta_j    = (r_{j+1}, r_{j+1}) / (r_j, r_j)
        p_{j+1}   = r_{j+1} + beta_j p_j

Arithmetic: fp64 vectors; the matrix-vector product is the oracle's own
definition SpMV (oracle/coo_spmv.c, long double accumulation, rounded to
fp64); dot products are numpy fp64 dots. No blocking, fusion or reordering
beyond the algorithm above.
"""
from __future__ import annotations

import numpy as np

from . import coo


def matvec(a, v: np.ndarray) -> np.ndarray:
    """A v by definition (COO, long double accumulation)."""
    y, _ = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val.astype(np.float64), np.asarray(v, np.float64), 1.0, 0.0, None)
    return y


def cg(a, b: np.ndarray, x0: np.ndarray, iters: int, keep_history: bool = False):
    """`iters` CG steps from x0 (no stopping test: the caller fixes the count).

    Returns (x, r, rr_history) where rr_history[j] = (r_j, r_j) for
    j = 0..iters; with keep_history also the lists of r_j and p_j."""
    b = np.asarray(b, np.float64)
    x = np.array(x0, np.float64)
    r = b - matvec(a, x)
    p = r.copy()
    rr = float(np.dot(r, r))
    hist = [rr]
    rs, ps = [r.copy()], [p.copy()]
    for _ in range(iters):
        if rr == 0.0:
            hist.append(0.0)
            continue
        q = matvec(a, p)
        alpha = rr / float(np.dot(p, q))
        x = x + alpha * p
        r = r - alpha * q
        rr_new = float(np.dot(r, r))
        beta = rr_new / rr
        p = r + beta * p
        rr = rr_new
        hist.append(rr)
        if keep_history:
            rs.append(r.copy())
            ps.append(p.copy())
    if keep_history:
        return x, r, np.array(hist), rs, ps
    return x, r, np.array(hist)
