"""ORACLE (test infrastructure only): analytic A*x for the FDM/FVM stencil
matrices the paper motivates CRSD with ("Once the FDM or
FVM is used, the coefficient matrix of discrete PDEs is usually the diagonal
sparse matrix"); SURVEY.md §8(c) "SpMV values, closed forms".

Matrix: grid n1 x n2 x n3, row = i + n1*(j + n2*k), couplings -1 to every
stencil neighbour inside the grid (Dirichlet truncation), diagonal c
(4, 6, 26 for 5/7/27-point). Write p_k = [g_k + 1 < n_k], m_k = [g_k >= 1]
for the neighbours that exist along dimension k.

Derivation (not a re-application of the stencil): (A x)_r = c x_r - sum_n x_n.
For x affine, x_n = x_r + sum_k b_k delta_k; for x = sum_k g_k^2,
x_n = x_r + sum_k (2 g_k delta_k + delta_k^2). The neighbour sums factor
per dimension:
  7/5-point (axis neighbours): |N| = sum_k (p_k + m_k),
      sum_n delta_k = p_k - m_k,  sum_n delta_k^2 = p_k + m_k.
  27-point (tensor neighbours): C_k = 1 + p_k + m_k, |N| = prod C_k - 1,
      sum_n delta_k = (p_k - m_k) prod_{l!=k} C_l,
      sum_n delta_k^2 = (p_k + m_k) prod_{l!=k} C_l.
Every value is an integer of magnitude < 2^24 at the BASELINE grid sizes,
hence exact in fp32 and fp64 in any summation order.
"""
from __future__ import annotations

import numpy as np


def _coords(dims, row_begin=0, row_end=None):
    dims = list(dims) + [1] * (3 - len(dims))
    n = dims[0] * dims[1] * dims[2]
    idx = np.arange(row_begin, n if row_end is None else row_end, dtype=np.int64)
    g = [idx % dims[0], (idx // dims[0]) % dims[1], idx // (dims[0] * dims[1])]
    p = [(g[k] + 1 < dims[k]).astype(np.int64) for k in range(3)]
    m = [(g[k] >= 1).astype(np.int64) for k in range(3)]
    return dims, g, p, m


def stencil_apply(dims, kind: str, xkind: str, coef=None, row_begin=0, row_end=None) -> np.ndarray:
    """Exact A*x (float64) for the Dirichlet stencil of ``kind`` and
    x = 'ones' | 'linear' (a + sum b_k g_k) | 'quadratic' (sum g_k^2),
    for rows [row_begin, row_end) (default: all)."""
    dims, g, p, m = _coords(dims, row_begin, row_end)
    if kind in ("5pt", "7pt"):
        c = 4 if kind == "5pt" else 6
        active = [0, 1] if kind == "5pt" else [0, 1, 2]
        N = sum(p[k] + m[k] for k in active)
        S1 = {k: p[k] - m[k] for k in active}
        S2 = {k: p[k] + m[k] for k in active}
    elif kind == "27pt":
        c = 26
        active = [0, 1, 2]
        C = [1 + p[k] + m[k] for k in range(3)]
        N = C[0] * C[1] * C[2] - 1
        S1 = {k: (p[k] - m[k]) * C[(k + 1) % 3] * C[(k + 2) % 3] for k in active}
        S2 = {k: (p[k] + m[k]) * C[(k + 1) % 3] * C[(k + 2) % 3] for k in active}
    else:
        raise ValueError(kind)
    if xkind == "ones":
        return (c - N).astype(np.float64)
    if xkind == "linear":
        a, b = coef if coef is not None else (3.0, (1.0, -2.0, 5.0))
        x = a + sum(b[k] * g[k] for k in range(3))
        return (c - N) * x - sum(b[k] * S1[k] for k in active)
    if xkind == "quadratic":
        x = sum(g[k] * g[k] for k in range(3))
        return ((c - N) * x - sum(2 * g[k] * S1[k] + S2[k] for k in active)).astype(np.float64)
    raise ValueError(xkind)


def interior_mask(dims) -> np.ndarray:
    dims, g, p, m = _coords(dims)
    ok = np.ones(g[0].shape, dtype=bool)
    for k in range(3):
        if dims[k] > 1:
            ok &= (p[k] == 1) & (m[k] == 1)
    return ok
