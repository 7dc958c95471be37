"""Seeded synthetic matrices (COO) and vectors with the shapes of the paper's workloads.

The paper evaluates on FDM/FVM diagonal sparse matrices (PAPER.md P:L65-79,
Table V) that are not available offline; SURVEY.md §8(d) replaces
them by the synthetic configurations C1-C5 of BASELINE.json. Every generator
is deterministic in its ``seed``. Random per-entry values are drawn with a
counter-based hash of (row, slot) so that a row range generated on one rank
equals the same rows of the global matrix (needed by the row-partitioned
multi-GPU path).

No CRSD arithmetic lives here.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Callable, Iterable, Optional, Sequence

import numpy as np

from . import fast as _fast

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


@dataclass
class COO:
    """A sparse matrix in coordinate form (int64 indices, float64/float32 values)."""

    nrows: int
    ncols: int
    row: np.ndarray
    col: np.ndarray
    val: np.ndarray

    @property
    def nnz(self) -> int:
        return int(self.row.shape[0])

    def astype(self, dtype) -> "COO":
        return COO(self.nrows, self.ncols, self.row, self.col, self.val.astype(dtype))

    def sorted(self) -> "COO":
        order = np.lexsort((self.col, self.row))
        return COO(self.nrows, self.ncols, self.row[order], self.col[order], self.val[order])

    def shuffled(self, seed: int) -> "COO":
        p = np.random.default_rng(seed).permutation(self.nnz)
        return COO(self.nrows, self.ncols, self.row[p], self.col[p], self.val[p])


# ---------------------------------------------------------------------------
# counter-based uniform numbers (splitmix64 finaliser), vectorised
# ---------------------------------------------------------------------------
def _splitmix64(z: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = (z + np.uint64(0x9E3779B97F4A7C15)) & _M64
        z = ((z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)) & _M64
        z = ((z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)) & _M64
        return z ^ (z >> np.uint64(31))


def counter_uniform(counter: np.ndarray, seed: int) -> np.ndarray:
    """U[0,1) (53-bit) from a counter array and a seed; range-independent."""
    c = counter.astype(np.uint64, copy=False)
    with np.errstate(over="ignore"):
        z = _splitmix64(c * np.uint64(0x2545F4914F6CDD1D) ^ np.uint64(seed & 0xFFFFFFFFFFFFFFFF))
    return (z >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


def nonzero_uniform(rng: np.random.Generator, n: int) -> np.ndarray:
    """n draws of U(-1,1) with exact zeros redrawn."""
    v = rng.uniform(-1.0, 1.0, n)
    while True:
        z = v == 0.0
        if not z.any():
            return v
        v[z] = rng.uniform(-1.0, 1.0, int(z.sum()))


# ---------------------------------------------------------------------------
# stencils on structured grids (FDM/FVM)
# ---------------------------------------------------------------------------
def _disps(kind: str):
    if kind == "5pt":
        return [(0, 0, 0), (1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0)]
    if kind == "7pt":
        return [(0, 0, 0), (1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0), (0, 0, 1), (0, 0, -1)]
    if kind == "27pt":
        return [(a, b, c) for c in (-1, 0, 1) for b in (-1, 0, 1) for a in (-1, 0, 1)]
    raise ValueError(kind)


def stencil(
    dims: Sequence[int],
    kind: str,
    *,
    center: str = "dirichlet",
    values: str = "exact",
    seed: int = 0,
    drop: Optional[Callable] = None,
    row_begin: int = 0,
    row_end: Optional[int] = None,
) -> COO:
    """Stencil matrix (see ``stencil_numpy``, the definition). Large grids go
    through gen/fastgen.c, which produces the same COO bit for bit
    (tests/test_gen.py); ``drop`` must then be a ``c3_drop`` mask."""
    d3 = [int(d) for d in list(dims) + [1] * (3 - len(dims))]
    if row_end is None:
        row_end = d3[0] * d3[1] * d3[2]
    if (row_end - row_begin) >= 200_000 and (drop is None or hasattr(drop, "c3_params")) and _fast.available():
        if center not in ("dirichlet", "present") or values not in ("exact", "random"):
            raise ValueError((center, values))
        disps = _disps(kind)
        lin = [di + d3[0] * (dj + d3[1] * dk) for (di, dj, dk) in disps]
        disps = [disps[q] for q in np.argsort(lin, kind="stable")]
        r, c, v = _fast.stencil(d3, disps, center == "present", values == "random", seed,
                                None if drop is None else drop.c3_params, row_begin, row_end)
        n = d3[0] * d3[1] * d3[2]
        return COO(n, n, r, c, v)
    return stencil_numpy(dims, kind, center=center, values=values, seed=seed, drop=drop, row_begin=row_begin,
                         row_end=row_end)


def stencil_numpy(
    dims: Sequence[int],
    kind: str,
    *,
    center: str = "dirichlet",
    values: str = "exact",
    seed: int = 0,
    drop: Optional[Callable] = None,
    row_begin: int = 0,
    row_end: Optional[int] = None,
) -> COO:
    """Stencil matrix on an n1 x n2 x n3 grid, row index = i + n1*(j + n2*k).

    Couplings are -1. ``center='dirichlet'`` puts the number of stencil
    neighbours on the diagonal (4, 6 or 26); ``center='present'`` puts the
    number of couplings present in that row (so A*1 == 0 in every row).
    ``values='random'`` multiplies every entry by (1 + 0.1*U(-1,1)) drawn
    from a counter hash of (row, slot) -- SURVEY.md §8(d) C2.
    ``drop(i, j, k, (di, dj, dk)) -> bool mask`` removes couplings (idle
    sections). Only rows [row_begin, row_end) are emitted.
    Output is sorted by (row, col).
    """
    dims = list(dims) + [1] * (3 - len(dims))
    n1, n2, n3 = (int(d) for d in dims)
    n = n1 * n2 * n3
    if row_end is None:
        row_end = n
    disps = _disps(kind)
    lin = [di + n1 * (dj + n2 * dk) for (di, dj, dk) in disps]
    order = np.argsort(lin, kind="stable")
    disps = [disps[q] for q in order]
    lin = np.array([lin[q] for q in order], dtype=np.int64)
    m = len(disps)
    idx = np.arange(row_begin, row_end, dtype=np.int64)
    i = idx % n1
    j = (idx // n1) % n2
    k = idx // (n1 * n2)
    valid = np.empty((idx.shape[0], m), dtype=bool)
    cq = None
    for q, (di, dj, dk) in enumerate(disps):
        v = (i + di >= 0) & (i + di < n1) & (j + dj >= 0) & (j + dj < n2) & (k + dk >= 0) & (k + dk < n3)
        if (di, dj, dk) == (0, 0, 0):
            cq = q
        elif drop is not None:
            v &= ~drop(i, j, k, (di, dj, dk))
        valid[:, q] = v
    vals = np.full((idx.shape[0], m), -1.0, dtype=np.float64)
    if center == "dirichlet":
        vals[:, cq] = float(m - 1)
    elif center == "present":
        vals[:, cq] = (valid.sum(axis=1) - 1).astype(np.float64)
    else:
        raise ValueError(center)
    if values == "random":
        ctr = idx[:, None] * np.int64(m) + np.arange(m, dtype=np.int64)[None, :]
        u = counter_uniform(ctr, seed)
        vals *= 1.0 + 0.1 * (2.0 * u - 1.0)
    elif values != "exact":
        raise ValueError(values)
    if center == "present":
        # a row without couplings has center 0: that is no nonzero at all
        # (an idle section of the main diagonal), so it is not emitted
        valid[:, cq] &= vals[:, cq] != 0.0
    cols = idx[:, None] + lin[None, :]
    rows = np.broadcast_to(idx[:, None], valid.shape)
    return COO(n, n, rows[valid], cols[valid], vals[valid])


def stencil_5pt(nx: int, ny: int, **kw) -> COO:
    return stencil((nx, ny, 1), "5pt", **kw)


def stencil_7pt(n1: int, n2: int, n3: int, **kw) -> COO:
    return stencil((n1, n2, n3), "7pt", **kw)


def stencil_27pt(n1: int, n2: int, n3: int, **kw) -> COO:
    return stencil((n1, n2, n3), "27pt", **kw)


def grid_coords(dims: Sequence[int], row_begin: int = 0, row_end: Optional[int] = None):
    dims = list(dims) + [1] * (3 - len(dims))
    n1, n2, n3 = dims
    if row_end is None:
        row_end = n1 * n2 * n3
    idx = np.arange(row_begin, row_end, dtype=np.int64)
    return idx % n1, (idx // n1) % n2, idx // (n1 * n2)


# ---------------------------------------------------------------------------
# scatter points (nonzeros alone on their diagonal)
# ---------------------------------------------------------------------------
def inject_scatter(
    a: COO,
    count: int,
    lo: int,
    hi: int,
    exclude_offsets: Iterable[int],
    seed: int,
    row_range: Optional[tuple] = None,
) -> COO:
    """Append ``count`` points: rows uniform, |offset| uniform in [lo, hi] with
    a random sign, offsets in ``exclude_offsets`` (the stencil's) and columns
    outside [0, ncols) redrawn, duplicate positions redrawn. Values U(-1,1)\\{0}.
    The appended entries are NOT merged in sorted order (the builder
    canonicalises). Whether a point ends up as a CRSD scatter point is the
    builder's decision, not the generator's.
    """
    rng = np.random.default_rng(seed)
    excl = np.array(sorted(set(int(e) for e in exclude_offsets)), dtype=np.int64)
    r0, r1 = (0, a.nrows) if row_range is None else row_range
    rows = np.empty(0, np.int64)
    cols = np.empty(0, np.int64)
    while rows.shape[0] < count:
        need = count - rows.shape[0]
        nd = int(need * 1.3) + 16
        r = rng.integers(r0, r1, nd, dtype=np.int64)
        mag = rng.integers(lo, hi + 1, nd, dtype=np.int64)
        sgn = np.where(rng.integers(0, 2, nd) == 0, -1, 1).astype(np.int64)
        off = mag * sgn
        c = r + off
        ok = (c >= 0) & (c < a.ncols)
        if excl.size:
            ok &= ~np.isin(off, excl)
        r, c = r[ok], c[ok]
        rows = np.concatenate([rows, r])
        cols = np.concatenate([cols, c])
        key = rows * np.int64(a.ncols) + cols
        _, first = np.unique(key, return_index=True)
        first.sort()
        rows, cols = rows[first], cols[first]
    rows, cols = rows[:count], cols[:count]
    vals = nonzero_uniform(rng, count)
    return COO(
        a.nrows,
        a.ncols,
        np.concatenate([a.row, rows]),
        np.concatenate([a.col, cols]),
        np.concatenate([a.val.astype(np.float64), vals]),
    )


# ---------------------------------------------------------------------------
# banded matrix with irregular offset groups (BASELINE.json config 4)
# ---------------------------------------------------------------------------
C4_GROUPS = [
    [-40003, -40002, -40001],
    [-9001],
    [-1201, -1200],
    [-333, -47],
    [-1, 0, 1],
    [47, 333],
    [1200, 1201],
    [9001],
    [40001, 40002, 40003],
]


def c4_ranges(n: int):
    """Row ranges and offset sets of config 4, scaled to n rows."""
    g = C4_GROUPS
    all19 = sorted(o for grp in g for o in grp)
    mid5 = sorted(o for grp in g[2:7] for o in grp)
    ad3 = sorted(g[0] + g[4] + g[8])
    last = [-9001, -333, -47, -1, 0, 1, 47, 333, 9001]
    b = [0, n * 23 // 100, n * 51 // 100, n * 74 // 100, n]
    return [(b[0], b[1], all19), (b[1], b[2], mid5), (b[2], b[3], ad3), (b[3], b[4], last)]


def band(n: int, ranges, seed: int, row_begin: int = 0, row_end: Optional[int] = None) -> COO:
    """Banded matrix (see ``band_numpy``, the definition); large row ranges
    through gen/fastgen.c, bit for bit the same (tests/test_gen.py)."""
    if row_end is None:
        row_end = n
    if row_end - row_begin >= 200_000 and _fast.available():
        r, c, v = _fast.band(n, ranges, seed, row_begin, row_end)
        return COO(n, n, r, c, v)
    return band_numpy(n, ranges, seed, row_begin, row_end)


def band_numpy(n: int, ranges, seed: int, row_begin: int = 0, row_end: Optional[int] = None) -> COO:
    """Banded matrix: rows [a,b) carry the offsets of their range; entries with
    columns outside [0,n) are omitted. Values U(-1,1)\\{0} from a counter hash
    of (row, offset) so row ranges agree with the global matrix."""
    if row_end is None:
        row_end = n
    R, C, V = [], [], []
    for a, b, offs in ranges:
        a2, b2 = max(a, row_begin), min(b, row_end)
        if a2 >= b2:
            continue
        offs = np.array(sorted(offs), dtype=np.int64)
        idx = np.arange(a2, b2, dtype=np.int64)
        cols = idx[:, None] + offs[None, :]
        valid = (cols >= 0) & (cols < n)
        ctr = idx[:, None] * np.int64(1 << 20) + (offs[None, :] + np.int64(1 << 19))
        u = counter_uniform(ctr, seed)
        v = 2.0 * u - 1.0
        v[v == 0.0] = 0.5
        R.append(np.broadcast_to(idx[:, None], valid.shape)[valid])
        C.append(cols[valid])
        V.append(v[valid])
    if not R:
        e = np.empty(0, np.int64)
        return COO(n, n, e, e.copy(), np.empty(0))
    return COO(n, n, np.concatenate(R), np.concatenate(C), np.concatenate(V))


# ---------------------------------------------------------------------------
# BASELINE.json configurations
# ---------------------------------------------------------------------------
def config1(values: str = "random") -> COO:
    """C1: 2D 5-pt (4/-1) on 64x64 plus 16 scatter points (seed 1), offsets in +-[65, 4095]."""
    a = stencil_5pt(64, 64, values=values, seed=1)
    stencil_offs = [0, 1, -1, 64, -64]
    return inject_scatter(a, 16, 65, 4095, stencil_offs, seed=1)


def config2(n: int = 256, values: str = "random", seed: int = 2, row_begin=0, row_end=None) -> COO:
    """C2: 3D 7-pt (6/-1) on n^3 (n=256: 16,777,216 rows, 117,047,296 nnz)."""
    return stencil_7pt(n, n, n, values=values, seed=seed, row_begin=row_begin, row_end=row_end)


def c3_drop(n: int):
    """Zeroed sub-blocks of C3 scaled to an n^3 grid (n=192 gives SURVEY.md §8(d) C3):
    B1 k in [n/4, n/3): drop the 9 dk=+1 couplings; B2 j in [n/3, 2n/3) x k in
    [n/2, 5n/6): drop the 18 dj=+-1 couplings; B3 k in [5n/6, 11n/12): drop all 26."""
    k1a, k1b = n * 48 // 192, n * 64 // 192
    j2a, j2b = n * 64 // 192, n * 128 // 192
    k2a, k2b = n * 96 // 192, n * 160 // 192
    k3a, k3b = n * 160 // 192, n * 176 // 192

    def drop(i, j, k, d):
        di, dj, dk = d
        m = np.zeros(i.shape, dtype=bool)
        if dk == 1:
            m |= (k >= k1a) & (k < k1b)
        if dj != 0:
            m |= (j >= j2a) & (j < j2b) & (k >= k2a) & (k < k2b)
        m |= (k >= k3a) & (k < k3b)
        return m

    drop.c3_params = (k1a, k1b, j2a, j2b, k2a, k2b, k3a, k3b)  # the same rule in gen/fastgen.c
    return drop


def config3(n: int = 192, values: str = "random", seed: int = 3, scatter_frac: float = 0.001) -> COO:
    """C3: 27-pt FVM stencil on n^3 with idle sections and 0.1% scatter (seed 3).
    Center = number of present couplings."""
    a = stencil_27pt(n, n, n, center="present", values=values, seed=seed, drop=c3_drop(n))
    ncoup = (3 * n - 2) ** 3
    nsc = int(round(ncoup * scatter_frac))
    st = sorted({di + n * (dj + n * dk) for dk in (-1, 0, 1) for dj in (-1, 0, 1) for di in (-1, 0, 1)})
    hi = 2 * n * n  # 73,728 at n=192
    if nsc:
        a = inject_scatter(a, nsc, 2, hi, st, seed=seed)
    return a


def config4(n: int = 100_000_000, seed: int = 4, row_begin=0, row_end=None) -> COO:
    """C4: banded, 19 offsets in 9 groups forming 4 patterns by row range."""
    return band(n, c4_ranges(n), seed, row_begin, row_end)


def config5(n: int = 768, values: str = "exact", seed: int = 5, row_begin=0, row_end=None) -> COO:
    """C5: 3D 7-pt (6/-1) on n^3 (n=768: 452,984,832 rows)."""
    return stencil_7pt(n, n, n, values=values, seed=seed, row_begin=row_begin, row_end=row_end)


# ---------------------------------------------------------------------------
# random diagonal matrices for property tests
# ---------------------------------------------------------------------------
def random_diagonal(
    nrows: int,
    ncols: int,
    seed: int,
    ndiag: int = 6,
    max_off: Optional[int] = None,
    p_break: float = 0.05,
    max_break: int = 8,
    n_scatter: int = 5,
    n_zeros: int = 0,
) -> COO:
    """Diagonals at random offsets (with adjacent runs), each broken by random
    zero runs, plus random scatter points and optionally explicit zeros."""
    rng = np.random.default_rng(seed)
    if max_off is None:
        max_off = max(1, min(nrows, ncols))
    offs = set()
    ndiag = min(ndiag, nrows + ncols - 1)
    tries = 0
    while len(offs) < ndiag and tries < 50 * ndiag:
        tries += 1
        o = int(rng.integers(-min(max_off, nrows - 1), min(max_off, ncols - 1) + 1))
        run = int(rng.integers(1, 4))
        for t in range(run):
            oo = o + t
            if -(nrows - 1) <= oo <= ncols - 1:
                offs.add(oo)
    R, C = [], []
    for o in sorted(offs):
        r = np.arange(max(0, -o), min(nrows, ncols - o), dtype=np.int64)
        keep = np.ones(r.shape[0], dtype=bool)
        t = 0
        while t < r.shape[0]:
            if rng.random() < p_break:
                ln = int(rng.integers(1, max_break + 1))
                keep[t : t + ln] = False
                t += ln
            else:
                t += 1
        R.append(r[keep])
        C.append(r[keep] + o)
    rows = np.concatenate(R) if R else np.empty(0, np.int64)
    cols = np.concatenate(C) if C else np.empty(0, np.int64)
    vals = nonzero_uniform(rng, rows.shape[0])
    a = COO(nrows, ncols, rows, cols, vals)
    if n_scatter:
        key = set((rows * ncols + cols).tolist())
        sr, sc = [], []
        tries = 0
        while len(sr) < n_scatter and tries < 100 * n_scatter:
            tries += 1
            r = int(rng.integers(0, nrows))
            c = int(rng.integers(0, ncols))
            if r * ncols + c in key:
                continue
            key.add(r * ncols + c)
            sr.append(r)
            sc.append(c)
        a = COO(
            nrows,
            ncols,
            np.concatenate([a.row, np.array(sr, np.int64)]),
            np.concatenate([a.col, np.array(sc, np.int64)]),
            np.concatenate([a.val, nonzero_uniform(rng, len(sr))]),
        )
    if n_zeros and a.nnz:
        z = rng.choice(a.nnz, size=min(n_zeros, a.nnz), replace=False)
        a.val[z] = np.where(rng.integers(0, 2, z.shape[0]) == 0, 0.0, -0.0)
    return a


def vectors(n: int, kind: str = "random", seed: int = 0, dims=None, coef=None) -> np.ndarray:
    """x / y0 vectors: 'random' U(-1,1); 'ones'; 'linear' a + sum_k b_k g_k and
    'quadratic' sum_k g_k^2 over grid coordinates g = (i, j, k) of ``dims``;
    'nan' (to check that beta == 0 never reads y)."""
    if kind == "random":
        return np.random.default_rng(seed).uniform(-1.0, 1.0, n)
    if kind == "ones":
        return np.ones(n)
    if kind == "nan":
        return np.full(n, np.nan)
    if kind in ("linear", "quadratic"):
        g = grid_coords(dims)
        if kind == "linear":
            a, b = coef if coef is not None else (3.0, (1.0, -2.0, 5.0))
            return a + b[0] * g[0] + b[1] * g[1] + b[2] * g[2]
        return (g[0] * g[0] + g[1] * g[1] + g[2] * g[2]).astype(np.float64)
    raise ValueError(kind)


# ---------------------------------------------------------------------------
# symmetric positive definite inputs for the CG iteration
# ---------------------------------------------------------------------------
def spd_stencil_scatter(dims: Sequence[int], kind: str = "7pt", n_pairs: int = 0, seed: int = 0, shift: float = 0.0) -> COO:
    """Dirichlet stencil (center = number of stencil neighbours, couplings -1:
    symmetric, irreducibly diagonally dominant => SPD) plus ``n_pairs``
    symmetric off-stencil pairs (r, c), (c, r) with one value v in U(-1,1)\\{0};
    each pair adds |v| to both diagonal entries (and ``shift`` to every
    diagonal entry), which keeps the matrix diagonally dominant, hence SPD.
    The pairs exercise the scatter-point path inside CG."""
    a = stencil(dims, kind)
    n = a.nrows
    rng = np.random.default_rng(seed)
    diag_add = np.full(n, float(shift))
    pr, pc, pv = [], [], []
    if n_pairs:
        taken = set((a.row * np.int64(n) + a.col).tolist())
        while len(pr) < n_pairs:
            r = int(rng.integers(0, n))
            c = int(rng.integers(0, n))
            if r == c or r * n + c in taken:
                continue
            taken.add(r * n + c)
            taken.add(c * n + r)
            v = float(nonzero_uniform(rng, 1)[0])
            pr += [r, c]
            pc += [c, r]
            pv += [v, v]
            diag_add[r] += abs(v)
            diag_add[c] += abs(v)
    val = a.val.astype(np.float64).copy()
    on_diag = a.row == a.col
    val[on_diag] += diag_add[a.row[on_diag]]
    return COO(
        n,
        n,
        np.concatenate([a.row, np.array(pr, np.int64)]),
        np.concatenate([a.col, np.array(pc, np.int64)]),
        np.concatenate([val, np.array(pv, np.float64)]),
    )
