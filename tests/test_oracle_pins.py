"""Pins of the oracle against what the paper and mathematics fix (CPU only).

Each oracle function is checked against something other than itself:
  crsd_ref      -- Fig. 2 -> Fig. 4 / Table III golden (P:L313-349, P:L449-465,
                   P:L503-511), grouping example,
                   DIA special case (P:L81-95 textbook DIA), presence-rule edge
                   cases worked by hand
  coo           -- coo_spmv: dense brute-force product (numpy longdouble),
                   scipy.sparse, stencil closed forms (exact integers);
                   rows_spmv: dense brute force on shuffled row samples (first,
                   last, empty rows; beta != 0), bitwise against coo_spmv,
                   closed forms; parity_error: hand-worked cases; coo_spmv_native:
                   summation bound vs the definition, thread-count invariance,
                   closed forms
  closed_forms  -- interior values stated in SURVEY.md §8(c) (0, 0, -4/-6/-54)
  decode        -- round trip of the paper-order construction, and corrupted
                   layouts that must be rejected
"""
import numpy as np
import pytest
import scipy.sparse as sp
from hypothesis import given, settings, strategies as st

import gen
from oracle import closed_forms, coo, crsd_ref, decode
from tests.conftest import fig2_value

pytestmark = pytest.mark.filterwarnings("ignore::DeprecationWarning")


# ---------------------------------------------------------------- Fig. 2 golden
@pytest.mark.parametrize("idle_max", [1, 2])
def test_fig2_golden(fig2, fig2_expected, idle_max):
    nrows, ncols, row, col, val, _ = fig2
    E = fig2_expected
    R = crsd_ref.build(nrows, ncols, row, col, val, mrows=E["mrows"], idle_max=idle_max)
    assert R.num_dia_patterns == E["num_dia_patterns"]
    assert [[list(g) for g in p] for p in R.matrix] == E["matrix"]
    assert R.offsets == E["offsets"]
    assert R.crsd_dia_index == E["crsd_dia_index"]
    assert R.NRS == E["NRS"] and R.NNzRS == E["NNzRS"] and R.SR == E["SR"] and R.NDias == E["NDias"]
    assert list(R.crsd_dia_val) == [fig2_value(n) for n in E["crsd_dia_val"]]
    # the only fill is the zero at v43 (flat index 18)
    assert np.flatnonzero(R.fill).tolist() == [18]
    assert R.num_scatter_rows == E["num_scatter_rows"]
    assert R.scatter_rowno == E["scatter_rowno"]
    assert R.num_scatter_width == E["num_scatter_width"]
    assert R.scatter_colval == E["scatter_colval"]
    assert R.scatter_val == [fig2_value(n) for n in E["scatter_val"]]
    segs = {str(s): [[lr, c, float(v)] for lr, c, v in lst] for s, lst in enumerate(R.seg_scatter) if lst}
    exp = {k: [[a, b, fig2_value(n)] for a, b, n in v] for k, v in E["b200_seg_scatter"].items()}
    assert segs == exp


def test_fig2_address_formula(fig2, fig2_expected):
    """P:L613-629 worked for group_id=2, p=1, d=1, local_id=0 (Appendix A)."""
    nrows, ncols, row, col, val, _ = fig2
    A = fig2_expected["address_example"]
    R = crsd_ref.build(nrows, ncols, row, col, val, mrows=2, idle_max=1)
    p, gid, d, lid = A["p"], A["group_id"], A["d"], A["local_id"]
    pre_nrs = sum(R.NRS[:p])
    loc = sum(R.NRS[i] * R.NNzRS[i] for i in range(p)) + (gid - pre_nrs) * R.NNzRS[p] + d * 2 + lid
    xi = R.Colv[p][d] + (gid - pre_nrs) * 2 + lid
    yi = R.SR[p] + (gid - pre_nrs) * 2 + lid
    assert (loc, xi, yi) == (A["value_index"], A["x_index"], A["y_index"])
    assert R.fill[loc] and R.crsd_dia_val[loc] == 0.0  # the filled v43


@pytest.mark.parametrize("idle_max,npat", [(0, 3), (3, None)])
def test_fig2_other_thresholds_do_not_reproduce_fig4(fig2, idle_max, npat):
    """idle_max=0 breaks the -1 diagonal (3 patterns); idle_max=3
    bridges the main diagonal through rows 2-4 (v55 is no longer scatter)."""
    nrows, ncols, row, col, val, _ = fig2
    R = crsd_ref.build(nrows, ncols, row, col, val, mrows=2, idle_max=idle_max)
    if npat is not None:
        assert R.num_dia_patterns == npat
    else:
        assert R.num_scatter_rows == 0


def test_grouping_example(fig2_expected):
    G = fig2_expected["grouping_example"]
    got = crsd_ref.groups(G["offsets"])
    assert [[t, list(g)] for t, g in got] == G["groups"]


def test_grouping_cases():
    # worked by hand from P:L281-297
    assert crsd_ref.pattern_repr([-1, 0, 1]) == [("AD", 3)]
    assert crsd_ref.pattern_repr([0, 1, 3, 4]) == [("AD", 2), ("AD", 2)]
    assert crsd_ref.pattern_repr([-5, 0, 5]) == [("NAD", 3)]
    assert crsd_ref.pattern_repr([-2, -1, 1]) == [("AD", 2), ("NAD", 1)]
    assert crsd_ref.pattern_repr([]) == []
    assert crsd_ref.pattern_repr([-9001, -333, -47, -1, 0, 1, 47, 333, 9001]) == [("NAD", 3), ("AD", 3), ("NAD", 3)]


# ------------------------------------------------------------ presence rule
def _present(entries, nrows, mrows, idle_max):
    return crsd_ref.present_sets(nrows, [(r, c, 1.0) for r, c in entries], mrows, idle_max)


def test_presence_isolated_point_is_scatter():
    p = _present([(5, 9)], 16, 4, 3)
    assert all(len(s) == 0 for s in p)


def test_presence_gap_equal_and_above_idle_max():
    # offset +2, nonzeros at rows 3 and 3+idle_max+1 (gap = idle_max zeros)
    m, im = 4, 2
    p = _present([(3, 5), (6, 8)], 16, m, im)  # gap rows 4,5 = 2 zeros -> bridged
    assert 2 in p[0] and 2 in p[1]
    p = _present([(3, 5), (7, 9)], 16, m, im)  # gap 3 zeros -> broken, both single
    assert 2 not in p[0] and 2 not in p[1]


def test_presence_two_in_segment_always_present():
    p = _present([(0, 0), (3, 3)], 8, 4, 0)  # gap 2 > idle_max 0, but cnt==2
    assert 0 in p[0]


def test_presence_empty_segment_bridged_only_if_idle_max_ge_mrows():
    ent = [(r, r) for r in range(0, 4)] + [(r, r) for r in range(8, 12)]
    p = _present(ent, 12, 4, 3)
    assert [0 in s for s in p] == [True, False, True]
    p = _present(ent, 12, 4, 4)
    assert [0 in s for s in p] == [True, True, True]


# ---------------------------------------------------------------- DIA special case
def test_single_segment_no_breaks_is_dia():
    """With mrows >= nrows and no idle sections, the CRSD value array is DIA's
    data[d*nrows + r] (Saad / Bell & Garland DIA)."""
    rng = np.random.default_rng(7)
    n = 40
    offs = [-7, -1, 0, 1, 3, 12]
    R_, C_, V_ = [], [], []
    dia = np.zeros((len(offs), n))
    for d, o in enumerate(offs):
        for r in range(n):
            c = r + o
            if 0 <= c < n:
                v = rng.uniform(0.5, 1.5)
                R_.append(r); C_.append(c); V_.append(v)
                dia[d, r] = v
    R = crsd_ref.build(n, n, np.array(R_), np.array(C_), np.array(V_), mrows=n, idle_max=n)
    assert R.num_dia_patterns == 1 and R.offsets[0] == offs
    assert np.array_equal(R.crsd_dia_val, dia.reshape(-1))
    assert R.num_scatter_rows == 0


# ---------------------------------------------------------------- decoder
@settings(max_examples=40, deadline=None)
@given(
    n=st.integers(1, 60),
    m=st.integers(1, 60),
    seed=st.integers(0, 10_000),
    mrows=st.sampled_from([1, 2, 3, 5, 32]),
    im=st.integers(-1, 6),
    nz=st.integers(0, 3),
)
def test_decode_roundtrip_of_reference(n, m, seed, mrows, im, nz):
    a = gen.random_diagonal(n, m, seed, ndiag=5, p_break=0.15, max_break=5, n_scatter=4, n_zeros=nz)
    R = crsd_ref.build(a.nrows, a.ncols, a.row, a.col, a.val, mrows=mrows, idle_max=im)
    L = crsd_ref.to_layout(R)
    decode.check_invariants(L, R.idle_max, a.nrows, a.ncols, a.row, a.col, a.val)


def test_decode_rejects_corruption(fig2):
    nrows, ncols, row, col, val, _ = fig2
    R = crsd_ref.build(nrows, ncols, row, col, val, mrows=2, idle_max=1)
    L = crsd_ref.to_layout(R)
    assert decode.roundtrip_equal(L, nrows, ncols, row, col, val)
    bad = dict(L, vals=L["vals"].copy())
    bad["vals"][3] = -bad["vals"][3]  # sign flip
    assert not decode.roundtrip_equal(bad, nrows, ncols, row, col, val)
    bad = dict(L, inst_offsets=[[0, 2, 3, 5, 7], [-2, 0, 1]])  # wrong offset
    assert not decode.roundtrip_equal(bad, nrows, ncols, row, col, val)
    bad = dict(L, vals=L["vals"].copy())
    bad["vals"][18] = -0.0  # a fill that is not +0.0 decodes as an entry
    assert not decode.roundtrip_equal(bad, nrows, ncols, row, col, val)
    bad = dict(L, inst_first_seg=np.array([0, 2]), inst_nseg=np.array([2, 1]))
    with pytest.raises(AssertionError):
        decode.check_invariants(bad, 1)


# ---------------------------------------------------------------- COO SpMV
def _dense_longdouble(a, x, alpha, beta, y0):
    A = np.zeros((a.nrows, a.ncols), dtype=np.longdouble)
    A[a.row, a.col] = a.val.astype(np.longdouble)
    y = np.longdouble(alpha) * (A @ x.astype(np.longdouble))
    if beta != 0:
        y = y + np.longdouble(beta) * y0.astype(np.longdouble)
    return y


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (-0.75, 0.5), (2.0, -1.25)])
def test_coo_spmv_vs_dense_bruteforce(seed, alpha, beta):
    rng = np.random.default_rng(seed)
    n, m = int(rng.integers(1, 64)), int(rng.integers(1, 64))
    a = gen.random_diagonal(n, m, seed, ndiag=6, n_scatter=6)
    x = rng.uniform(-1, 1, m)
    y0 = rng.uniform(-1, 1, n)
    y, s = coo.coo_spmv(n, m, a.row, a.col, a.val, x, alpha, beta, y0)
    ref = _dense_longdouble(a, x, alpha, beta, y0)
    assert np.array_equal(y, ref.astype(np.float64)) or np.max(np.abs(y - ref.astype(np.float64))) <= 1e-15 * max(1.0, np.max(s))


def test_coo_spmv_f32_vs_dense():
    rng = np.random.default_rng(11)
    a = gen.random_diagonal(50, 50, 11, ndiag=7, n_scatter=5).astype(np.float32)
    x = rng.uniform(-1, 1, 50).astype(np.float32)
    y0 = rng.uniform(-1, 1, 50).astype(np.float32)
    y, s = coo.coo_spmv(50, 50, a.row, a.col, a.val, x, -0.75, 0.5, y0)
    A = np.zeros((50, 50), dtype=np.longdouble)
    A[a.row, a.col] = a.val.astype(np.longdouble)
    ref = np.longdouble(-0.75) * (A @ x.astype(np.longdouble)) + np.longdouble(0.5) * y0.astype(np.longdouble)
    assert np.max(np.abs(y - ref.astype(np.float64))) <= 1e-15


def test_coo_spmv_vs_scipy():
    a = gen.config1()
    x = gen.vectors(a.ncols, "random", seed=5)
    y, s = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x)
    ref = sp.csr_matrix((a.val, (a.row, a.col)), shape=(a.nrows, a.ncols)) @ x
    assert coo.parity_error(ref, y, s) <= 1e-14


def test_coo_spmv_beta_zero_never_reads_y():
    a = gen.config1()
    x = gen.vectors(a.ncols, "random", seed=5)
    y, _ = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x, 1.0, 0.0, np.full(a.nrows, np.nan))
    assert np.all(np.isfinite(y))


def test_coo_spmv_rejects_out_of_range():
    with pytest.raises(ValueError):
        coo.coo_spmv(2, 2, np.array([0]), np.array([2]), np.array([1.0]), np.ones(2))


# ---------------------------------------------------------------- rows_spmv (sampled rows)
def _csr(a):
    """Row-sorted copy and its row pointer (the layout rows_spmv reads)."""
    order = np.lexsort((a.col, a.row))
    r, c, v = a.row[order], a.col[order], a.val[order]
    ptr = np.zeros(a.nrows + 1, np.int64)
    ptr[1:] = np.cumsum(np.bincount(r, minlength=a.nrows))
    return r, c, v, ptr


@pytest.mark.parametrize("seed", range(5))
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (-0.75, 0.5)])
def test_rows_spmv_vs_dense_bruteforce(seed, alpha, beta):
    """rows_spmv on a shuffled row subset (first and last rows and rows with no
    entries included) against the dense long-double product: a row_ptr
    off-by-one, or y0 indexed by the sample position instead of the row,
    fails here."""
    rng = np.random.default_rng(100 + seed)
    n, m = int(rng.integers(8, 64)), int(rng.integers(8, 64))
    a = gen.random_diagonal(n, m, seed, ndiag=5, n_scatter=4)
    # empty out a few rows entirely
    empty = rng.choice(n, size=3, replace=False)
    keep = ~np.isin(a.row, empty)
    a = gen.COO(n, m, a.row[keep], a.col[keep], a.val[keep])
    r, c, v, ptr = _csr(a)
    x = rng.uniform(-1, 1, m)
    y0 = rng.uniform(-1, 1, n)
    sel = np.unique(np.concatenate([[0, n - 1], empty, rng.integers(0, n, 10)]))
    sel = sel[rng.permutation(sel.shape[0])]  # sample order != row order
    y, sc = coo.rows_spmv(sel, ptr, c, v, x, alpha, beta, y0)
    ref = _dense_longdouble(a, x, alpha, beta, y0).astype(np.float64)
    assert np.max(np.abs(y - ref[sel])) <= 1e-15 * max(1.0, float(np.max(sc)))
    # rows without entries: beta * y0[row] exactly
    for t, row in enumerate(sel):
        if row in empty:
            assert y[t] == (beta * y0[row] if beta != 0 else 0.0)


def test_rows_spmv_equals_full_definition_bitwise():
    """Same entries in the same order: rows_spmv must give the full
    coo_spmv's bits for every sampled row (incl. scale)."""
    a = gen.config3(n=16)
    r, c, v, ptr = _csr(a)
    rng = np.random.default_rng(3)
    x = rng.uniform(-1, 1, a.ncols)
    y0 = rng.uniform(-1, 1, a.nrows)
    yf, sf = coo.coo_spmv(a.nrows, a.ncols, r, c, v, x, -0.75, 0.5, y0)
    sel = np.concatenate([[a.nrows - 1, 0], rng.integers(0, a.nrows, 300)])
    y, s2 = coo.rows_spmv(sel, ptr, c, v, x, -0.75, 0.5, y0)
    assert np.array_equal(y, yf[sel]) and np.array_equal(s2, sf[sel])


def test_rows_spmv_closed_form():
    """Sampled rows of the 7-point stencil applied to the quadratic vector:
    -6 in the interior, the closed form everywhere (exact integers)."""
    dims = (11, 9, 7)
    a = gen.stencil(dims, "7pt", values="exact")
    r, c, v, ptr = _csr(a)
    x = gen.vectors(a.ncols, "quadratic", dims=dims)
    sel = np.arange(a.nrows)[::-3]
    y, _ = coo.rows_spmv(sel, ptr, c, v, x)
    assert np.array_equal(y, closed_forms.stencil_apply(dims, "7pt", "quadratic")[sel])


# ---------------------------------------------------------------- parity_error
def test_parity_error_hand_cases():
    """The pass criterion of SURVEY.md §8(c): max over rows (not mean) of
    |y - y_ref| / scale; rows with scale 0 must match exactly; NaN fails."""
    ref = np.array([1.0, -2.0, 0.0, 4.0])
    scale = np.array([1.0, 2.0, 0.0, 8.0])
    assert coo.parity_error(ref.copy(), ref, scale) == 0.0
    y = ref + np.array([1e-13, 0.0, 0.0, 0.0])
    assert coo.parity_error(y, ref, scale) == pytest.approx(1e-13, rel=1e-3)
    y = ref + np.array([1e-13, 4e-13, 0.0, 8e-13])  # per-row 1e-13, 2e-13, -, 1e-13: max, not mean
    assert coo.parity_error(y, ref, scale) == pytest.approx(2e-13, rel=1e-3)
    y = ref.copy()
    y[2] = 1e-300  # a scale-0 row off by anything is a failure
    assert coo.parity_error(y, ref, scale) == float("inf")
    y = ref.copy()
    y[1] = np.nan
    assert coo.parity_error(y, ref, scale) == float("inf")
    assert coo.parity_error(np.zeros(2), np.zeros(2), np.zeros(2)) == 0.0
    # relative to the row's own scale: a large error on a large-scale row passes
    assert coo.parity_error(np.array([1e6 + 1e-7]), np.array([1e6]), np.array([1e6])) <= 1e-12


# ---------------------------------------------------------------- native-dtype baseline
@pytest.mark.parametrize("dt", [np.float64, np.float32])
@pytest.mark.parametrize("seed", range(4))
def test_coo_native_within_summation_bound_and_thread_invariant(dt, seed):
    """coo_spmv_native (the timed CPU baseline) against the long-double
    definition: per row |y - y_ref| <= (k + 2) u scale (k entries, u the unit
    roundoff; the recursive-summation bound), and the same bits for 1, 2, 3
    and 8 threads (each row is summed by one thread in entry order)."""
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 4000))
    a = gen.random_diagonal(n, n, seed, ndiag=9, n_scatter=30).astype(dt)
    keep = ~np.isin(a.row, rng.choice(n, size=min(n, 5), replace=False))  # some empty rows
    a = gen.COO(n, n, a.row[keep], a.col[keep], a.val[keep])
    r, c, v, ptr = _csr(a)
    x = rng.uniform(-1, 1, n).astype(dt)
    y0 = rng.uniform(-1, 1, n).astype(dt)
    for alpha, beta in ((1.0, 0.0), (-0.75, 0.5)):
        yref, sc = coo.coo_spmv(n, n, r, c, v, x, alpha, beta, y0)
        u = 2.0**-53 if dt == np.float64 else 2.0**-24
        k = np.diff(ptr).astype(np.float64)
        outs = [coo.coo_spmv_native(n, r, c, v, x, alpha, beta, y0, nthreads=t) for t in (1, 2, 3, 8)]
        assert outs[0].dtype == dt
        err = np.abs(outs[0].astype(np.float64) - yref)
        assert np.all(err <= (k + 2) * u * sc + (sc == 0) * 0.0)
        for o in outs[1:]:
            assert np.array_equal(o, outs[0])
    # beta == 0 never reads y0
    y = coo.coo_spmv_native(n, r, c, v, x, 1.0, 0.0, np.full(n, np.nan, dt), nthreads=3)
    assert np.all(np.isfinite(y))


def test_coo_native_closed_form_and_rejects_unsorted():
    dims = (13, 11, 9)
    a = gen.stencil(dims, "7pt", values="exact")
    x = gen.vectors(a.ncols, "linear", dims=dims)
    y = coo.coo_spmv_native(a.nrows, a.row, a.col, a.val, x, nthreads=4)
    assert np.array_equal(y, closed_forms.stencil_apply(dims, "7pt", "linear"))
    with pytest.raises(ValueError):
        coo.coo_spmv_native(2, np.array([1, 0]), np.array([0, 0]), np.array([1.0, 1.0]), np.ones(2))


# ---------------------------------------------------------------- closed forms
STENCILS = [("5pt", (17, 13, 1)), ("7pt", (9, 7, 5)), ("27pt", (7, 6, 5))]


@pytest.mark.parametrize("kind,dims", STENCILS)
@pytest.mark.parametrize("xkind", ["ones", "linear", "quadratic"])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_coo_spmv_matches_closed_form(kind, dims, xkind, dtype):
    a = gen.stencil(dims, kind, values="exact").astype(dtype)
    x = gen.vectors(a.ncols, xkind, dims=dims).astype(dtype)
    y, _ = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x)
    assert np.array_equal(y, closed_forms.stencil_apply(dims, kind, xkind))


@pytest.mark.parametrize("kind,dims,quad", [("5pt", (17, 13, 1), -4), ("7pt", (9, 7, 5), -6), ("27pt", (7, 6, 5), -54)])
def test_closed_form_interior_values(kind, dims, quad):
    """interior A*1 = 0, A*(affine) = 0, A*(sum g^2) = -4/-6/-54."""
    mask = closed_forms.interior_mask(dims)
    assert mask.any()
    assert np.all(closed_forms.stencil_apply(dims, kind, "ones")[mask] == 0)
    assert np.all(closed_forms.stencil_apply(dims, kind, "linear")[mask] == 0)
    assert np.all(closed_forms.stencil_apply(dims, kind, "quadratic")[mask] == quad)


def test_closed_form_boundary_ones():
    """Boundary A*1: number of boundary dimensions (7-pt), 27 - prod c_k (27-pt)."""
    y = closed_forms.stencil_apply((4, 4, 4), "7pt", "ones")
    assert y[0] == 3 and y[1] == 2 and y[1 + 4 + 16] == 0
    y = closed_forms.stencil_apply((4, 4, 4), "27pt", "ones")
    assert y[0] == 27 - 8 and y[1] == 27 - 12 and y[1 + 4] == 27 - 18 and y[1 + 4 + 16] == 0


def test_c3_present_center_rows_sum_to_zero():
    a = gen.config3(n=12, values="exact", scatter_frac=0.0)
    y, _ = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, np.ones(a.ncols))
    assert np.all(y == 0)


def test_paper_ell_rows_fig2_exact(fig2):
    """Fig. 2's scatter row 5 (scatter_rowno [5], colval [3,4,5,6])
    computed by the paper's ELL part equals the row's dot product exactly
    (small integers: every partial sum is exact)."""
    n, m, r, c, v, _ = fig2
    R = crsd_ref.build(n, m, r, c, v, mrows=2, idle_max=1)
    x = np.arange(1, m + 1, dtype=np.float64)
    out = crsd_ref.paper_ell_rows(R, x)
    assert list(out) == [5]
    row5 = [(cc, vv) for rr, cc, vv in zip(r, c, v) if rr == 5]
    assert out[5] == sum(vv * x[cc] for cc, vv in row5)


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_paper_ell_rows_match_definition(dt):
    """On random diagonal matrices with scatter points, the paper-order row
    products of the scatter rows agree with the definition within the
    recursive-summation bound (k u scale)."""
    a = gen.random_diagonal(300, 280, 4, ndiag=6, n_scatter=40).astype(dt)
    R = crsd_ref.build(a.nrows, a.ncols, a.row, a.col, a.val, mrows=32)
    x = np.random.default_rng(5).uniform(-1, 1, a.ncols).astype(dt)
    out = crsd_ref.paper_ell_rows(R, x, alpha=-0.75, dtype=dt)
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x, -0.75, 0.0, None)
    assert len(out) == R.num_scatter_rows > 0
    u = np.finfo(dt).eps
    for row, val in out.items():
        k = R.num_scatter_width + 2
        assert abs(float(val) - yref[row]) <= k * u * scale[row]
