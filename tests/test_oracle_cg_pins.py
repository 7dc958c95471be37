"""Pins of the CG oracle (oracle/cg_ref.py) against what the mathematics fixes,
not against a retyping of the algorithm (-m "not gpu"):

* finite termination: for SPD A of order n, CG reaches the exact solution in
  <= n steps in exact arithmetic (Hestenes & Stiefel 1952; Saad Thm 6.6) --
  checked against the closed-form solution of the 1D Dirichlet Laplacian
  tridiag(-1, 2, -1) x = 1, x_i = i (n + 1 - i) / 2 (i = 1..n), and against
  a dense LAPACK solve for a random SPD banded matrix;
* the first step is the steepest-descent step x_1 = x_0 + (r0.r0 / r0.A r0) r0;
* r_0 an eigenvector of A => convergence in one step (x_1 exact);
* residual orthogonality (r_i, r_j) = 0 and A-conjugacy (p_i, A p_j) = 0,
  i != j (Saad Prop. 6.13);
* the recurrence residual equals the true residual b - A x_j.
A dropped term, a wrong sign or a swapped alpha/beta fails one of these.
"""
import numpy as np
import pytest

import gen
from oracle import cg_ref


def _tridiag(n):
    r = np.concatenate([np.arange(n), np.arange(1, n), np.arange(n - 1)])
    c = np.concatenate([np.arange(n), np.arange(n - 1), np.arange(1, n)])
    v = np.concatenate([np.full(n, 2.0), np.full(n - 1, -1.0), np.full(n - 1, -1.0)])
    return gen.COO(n, n, r.astype(np.int64), c.astype(np.int64), v)


def _dense(a):
    d = np.zeros((a.nrows, a.ncols))
    d[a.row, a.col] = a.val
    return d


def _spd_band(n, seed):
    """Random symmetric banded matrix made SPD by diagonal dominance."""
    rng = np.random.default_rng(seed)
    rows, cols, vals = [], [], []
    offs = [1, 2, 5, 9]
    off_vals = {}
    for o in offs:
        v = rng.uniform(-1, 1, n - o)
        off_vals[o] = v
        i = np.arange(n - o)
        rows += [i, i + o]
        cols += [i + o, i]
        vals += [v, v]
    diag = np.full(n, 0.5)
    for o, v in off_vals.items():
        diag[: n - o] += np.abs(v)
        diag[o:] += np.abs(v)
    rows.append(np.arange(n))
    cols.append(np.arange(n))
    vals.append(diag)
    return gen.COO(n, n, np.concatenate(rows).astype(np.int64), np.concatenate(cols).astype(np.int64), np.concatenate(vals))


@pytest.mark.parametrize("n", [1, 2, 7, 40])
def test_cg_1d_laplacian_closed_form(n):
    a = _tridiag(n)
    i = np.arange(1, n + 1, dtype=np.float64)
    x_exact = i * (n + 1 - i) / 2.0
    x, r, hist = cg_ref.cg(a, np.ones(n), np.zeros(n), n)
    assert np.max(np.abs(x - x_exact)) <= 1e-10 * np.max(x_exact)
    assert np.sqrt(hist[-1]) <= 1e-10 * np.sqrt(n)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_cg_random_spd_vs_dense_solve(seed):
    n = 30
    a = _spd_band(n, seed)
    d = _dense(a)
    assert np.allclose(d, d.T) and np.min(np.linalg.eigvalsh(d)) > 0
    rng = np.random.default_rng(seed + 10)
    b = rng.uniform(-1, 1, n)
    x0 = rng.uniform(-1, 1, n)
    x, r, hist = cg_ref.cg(a, b, x0, n)
    xs = np.linalg.solve(d, b)
    assert np.max(np.abs(x - xs)) <= 1e-9 * np.max(np.abs(xs))


def test_cg_first_step_is_steepest_descent():
    a = _spd_band(25, 3)
    d = _dense(a)
    rng = np.random.default_rng(4)
    b, x0 = rng.uniform(-1, 1, 25), rng.uniform(-1, 1, 25)
    r0 = b - d @ x0
    x1_expected = x0 + (r0 @ r0) / (r0 @ d @ r0) * r0
    x1, r1, hist = cg_ref.cg(a, b, x0, 1)
    assert np.max(np.abs(x1 - x1_expected)) <= 1e-13 * np.max(np.abs(x1_expected))
    assert hist[0] == pytest.approx(r0 @ r0, rel=1e-14)
    assert hist[1] == pytest.approx(np.dot(b - d @ x1, b - d @ x1), rel=1e-9)


def test_cg_eigenvector_residual_converges_in_one_step():
    # tridiag(-1,2,-1): eigenvectors sin(k pi i / (n+1)), eigenvalues 2 - 2 cos(k pi / (n+1))
    n, k = 20, 3
    a = _tridiag(n)
    i = np.arange(1, n + 1)
    v = np.sin(k * np.pi * i / (n + 1))
    lam = 2 - 2 * np.cos(k * np.pi / (n + 1))
    x_true = np.random.default_rng(5).uniform(-1, 1, n)
    b = _dense(a) @ x_true
    x0 = x_true - v / lam  # r0 = A (x_true - x0) = v
    x1, r1, hist = cg_ref.cg(a, b, x0, 1)
    assert np.max(np.abs(x1 - x_true)) <= 1e-12
    assert hist[1] <= 1e-24 * hist[0] + 1e-28


def test_cg_orthogonality_and_conjugacy():
    n = 30
    a = _spd_band(n, 6)
    d = _dense(a)
    rng = np.random.default_rng(7)
    b, x0 = rng.uniform(-1, 1, n), np.zeros(n)
    x, r, hist, rs, ps = cg_ref.cg(a, b, x0, 8, keep_history=True)
    for i in range(len(rs)):
        for j in range(i):
            assert abs(rs[i] @ rs[j]) <= 1e-10 * np.linalg.norm(rs[i]) * np.linalg.norm(rs[j]) + 1e-300
            assert abs(ps[i] @ d @ ps[j]) <= 1e-10 * np.linalg.norm(ps[i]) * np.linalg.norm(d @ ps[j]) + 1e-300
    # the recurrence residual is the true residual
    assert np.max(np.abs(r - (b - d @ x))) <= 1e-12 * np.max(np.abs(b))
    assert hist[-1] == pytest.approx(r @ r, rel=1e-12)


def test_cg_stops_cleanly_at_exact_solution():
    a = _tridiag(5)
    b = _dense(a) @ np.ones(5)
    x, r, hist = cg_ref.cg(a, b, np.ones(5), 3)
    assert np.all(x == 1.0) and np.all(hist == 0.0)
