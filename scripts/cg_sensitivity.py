#!/usr/bin/env python
"""Tolerance evidence for the CG parity tests.

Runs the textbook CG twice on the CG test matrices: once as the oracle
(oracle/cg_ref.py: definition SpMV in long double, numpy fp64 dots) and once
with another admissible evaluation order (scipy CSR SpMV, vectors in the
matrix precision, dots in fp64 -- the GPU path's arithmetic), and prints the
largest relative differences of (r_j, r_j) and of x after K steps.
usage: python scripts/cg_sensitivity.py [K]
"""
import os
import sys

import numpy as np
import scipy.sparse as sp

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
from oracle import cg_ref  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 60
FLOOR = {np.float64: 1e-20, np.float32: 1e-8}
CASES = {
    "7pt": gen.spd_stencil_scatter((40, 40, 40), "7pt"),
    "27pt": gen.spd_stencil_scatter((24, 24, 24), "27pt"),
    "7pt+scatter": gen.spd_stencil_scatter((30, 30, 30), "7pt", n_pairs=500, seed=3),
    "5pt-ragged": gen.spd_stencil_scatter((61, 67), "5pt", n_pairs=40, seed=4),
}


def cg_other(A, b, x0, dt, k):
    A = A.astype(dt)
    x = x0.astype(dt)
    r = (b.astype(dt) - A @ x).astype(dt)
    p = r.copy()
    rr = float(np.dot(r.astype(np.float64), r.astype(np.float64)))
    h = [rr]
    for _ in range(k):
        q = (A @ p).astype(dt)
        al = rr / float(np.dot(p.astype(np.float64), q.astype(np.float64)))
        x = (x + dt(al) * p).astype(dt)
        r = (r - dt(al) * q).astype(dt)
        rn = float(np.dot(r.astype(np.float64), r.astype(np.float64)))
        p = (r + dt(rn / rr) * p).astype(dt)
        rr = rn
        h.append(rr)
    return x, np.array(h)


for name, a in CASES.items():
    n = a.nrows
    rng = np.random.default_rng(11)
    b = rng.uniform(-1, 1, n)
    x0 = rng.uniform(-0.5, 0.5, n)
    for dt in (np.float64, np.float32):
        ad = a.astype(dt)
        bq, xq = b.astype(dt).astype(np.float64), x0.astype(dt).astype(np.float64)
        xr, _, hr = cg_ref.cg(ad, bq, xq, K)
        A = sp.csr_matrix((ad.val, (ad.row, ad.col)), shape=(n, n))
        x, h = cg_other(A, bq, xq, dt, K)
        live = hr / hr[0] >= FLOOR[dt]
        print(f"{name:12s} {np.dtype(dt).name:8s} K={K} rr rel max {np.max(np.abs(h[live] - hr[live]) / hr[live]):.2e}"
              f"  x rel {np.max(np.abs(x - xr)) / np.max(np.abs(xr)):.2e}  rr_K/rr_0 {hr[-1] / hr[0]:.1e}")
