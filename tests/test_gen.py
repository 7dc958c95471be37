"""gen/fastgen.c (the C generators the benchmarks use for the 10^8-10^9-entry
BASELINE matrices) must produce the numpy generators' COO bit for bit: same
entries, same order, same value bits. CPU only."""
import numpy as np
import pytest

from gen import fast, matrices

pytestmark = pytest.mark.filterwarnings("ignore::DeprecationWarning")


def _same(a, r, c, v):
    assert np.array_equal(a.row, r) and np.array_equal(a.col, c)
    assert np.array_equal(a.val.view(np.uint64), v.view(np.uint64))


def _fast_stencil(dims, kind, center, values, seed, drop, rb, re):
    d3 = list(dims) + [1] * (3 - len(dims))
    disps = matrices._disps(kind)
    lin = [di + d3[0] * (dj + d3[1] * dk) for (di, dj, dk) in disps]
    disps = [disps[q] for q in np.argsort(lin, kind="stable")]
    return fast.stencil(d3, disps, center == "present", values == "random", seed,
                        None if drop is None else drop.c3_params, rb, re, nthreads=3)


@pytest.mark.parametrize("kind,dims", [("5pt", (23, 17, 1)), ("7pt", (13, 11, 9)), ("27pt", (9, 8, 7))])
@pytest.mark.parametrize("center", ["dirichlet", "present"])
@pytest.mark.parametrize("values", ["exact", "random"])
@pytest.mark.parametrize("rng_", [(0, None), (37, 400)])
def test_fast_stencil_equals_numpy(kind, dims, center, values, rng_):
    rb, re = rng_
    a = matrices.stencil_numpy(dims, kind, center=center, values=values, seed=7, row_begin=rb, row_end=re)
    r, c, v = _fast_stencil(dims, kind, center, values, 7, None, rb, re if re is not None else int(np.prod(dims)))
    _same(a, r, c, v)


@pytest.mark.parametrize("n", [24, 36])
@pytest.mark.parametrize("values", ["exact", "random"])
def test_fast_c3_stencil_equals_numpy(n, values):
    """The C3 idle blocks (c3_drop) and center = present couplings (rows whose
    couplings are all dropped have no entry at all)."""
    drop = matrices.c3_drop(n)
    a = matrices.stencil_numpy((n, n, n), "27pt", center="present", values=values, seed=3, drop=drop)
    r, c, v = _fast_stencil((n, n, n), "27pt", "present", values, 3, drop, 0, n**3)
    _same(a, r, c, v)


@pytest.mark.parametrize("rb,re", [(0, 300_000), (51_234, 177_777)])
def test_fast_band_equals_numpy(rb, re):
    n = 300_000
    ranges = matrices.c4_ranges(n)
    a = matrices.band_numpy(n, ranges, 4, rb, re)
    r, c, v = fast.band(n, ranges, 4, rb, re, nthreads=3)
    _same(a, r, c, v)


def test_dispatch_uses_fast_path_for_large_grids():
    """stencil()/band() switch to C above 200k rows; the result is the same
    matrix the numpy definition gives (spot-checked on a row block)."""
    a = matrices.stencil((64, 64, 64), "7pt", values="random", seed=2, row_begin=10_000, row_end=260_000)
    b = matrices.stencil_numpy((64, 64, 64), "7pt", values="random", seed=2, row_begin=10_000, row_end=260_000)
    _same(b, a.row, a.col, a.val)


@pytest.mark.parametrize("kind", ["band", "c3", "7pt"])
def test_fast_csr_mode_matches_coo(kind):
    """csr=True returns row pointers over the requested rows, consistent with
    the COO rows (rows without entries included)."""
    if kind == "band":
        n = 300_000
        ranges = [(1000, 90_000, [-5, 0, 7]), (120_000, 250_000, [-1, 0, 1, 40_000])]  # gaps: empty rows
        r, c, v = fast.band(n, ranges, 4, 500, 260_000, nthreads=2)
        p, c2, v2 = fast.band(n, ranges, 4, 500, 260_000, nthreads=2, csr=True)
        rb, re = 500, 260_000
    else:
        nn = 24
        drop = matrices.c3_drop(nn) if kind == "c3" else None
        st = "27pt" if kind == "c3" else "7pt"
        d3 = [nn, nn, nn]
        disps = matrices._disps(st)
        lin = [di + d3[0] * (dj + d3[1] * dk) for (di, dj, dk) in disps]
        disps = [disps[q] for q in np.argsort(lin, kind="stable")]
        rb, re = 100, nn**3 - 7
        args = (d3, disps, kind == "c3", True, 3, None if drop is None else drop.c3_params, rb, re)
        r, c, v = fast.stencil(*args, nthreads=2)
        p, c2, v2 = fast.stencil(*args, nthreads=2, csr=True)
    assert np.array_equal(c, c2) and np.array_equal(v, v2)
    expect = np.zeros(re - rb + 1, np.int64)
    expect[1:] = np.cumsum(np.bincount(r - rb, minlength=re - rb))
    assert np.array_equal(p, expect)
