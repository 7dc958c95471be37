"""GPU parity of crsd_spmv (C-ABI, sm_100a kernels) against the oracle.

Pass criterion (BASELINE.json north_star):
    max_r |y - y_ref| / scale_r <= 1e-12 (fp64), 1e-5 (fp32),
    scale_r = |alpha| sum_c |a_rc x_c| + |beta| |y0_r|; rows with scale 0 exact.
Derivation of the bound: the kernel accumulates each
row with k fused multiply-adds, plus the alpha/beta epilogue; the recursive
summation error is <= (k + 2) u scale_r with u = 2^-53 / 2^-24. For k <= 40
(27-point stencil + scatter) that is 4.7e-15 (fp64) and 2.5e-6 (fp32), under
the stated tolerances.
Closed-form checks (exact integers) are compared with ==.
"""
import os

import numpy as np
import pytest

import gen
from oracle import closed_forms, coo
from tests.conftest import have_gpu

pytestmark = pytest.mark.gpu

TOL = {np.float64: 1e-12, np.float32: 1e-5}
VARIANTS = [1, 2, 3, 4]  # CRSD_VARIANT_LDG, _TMA, _PIPE, _JIT

_CACHE = {}


def cached(name, fn, *args, **kw):
    """Full-size generators take seconds; share one instance per module."""
    key = (name, args, tuple(sorted(kw.items())))
    if key not in _CACHE:
        _CACHE[key] = fn(*args, **kw)
    return _CACHE[key]


@pytest.fixture(scope="module")
def torch_cuda():
    import torch

    if not torch.cuda.is_available():
        pytest.fail("no CUDA device: -m gpu tests need a B200")
    return torch


def _mat(a, **kw):
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, CRSDError

    try:
        return CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, **kw)
    except CRSDError as e:
        # the JIT codelets need a whole segment per CTA (staging <= 200 KB)
        if kw.get("variant") == 4 and "UNSUPPORTED" in str(e):
            pytest.skip(f"JIT variant not applicable: {e}")
        raise


def _run(torch, A, x, alpha=1.0, beta=0.0, y0=None, nrows=None):
    dt = torch.float64 if A.dtype == np.float64 else torch.float32
    xd = torch.from_numpy(np.ascontiguousarray(x)).to("cuda", dt)
    if y0 is None:
        yd = torch.full((nrows,), float("nan"), device="cuda", dtype=dt)
    else:
        yd = torch.from_numpy(np.ascontiguousarray(y0)).to("cuda", dt)
    A.spmv(xd, yd, alpha, beta)
    torch.cuda.synchronize()
    return yd.cpu().numpy()


def _parity(torch, a, dt, alpha=1.0, beta=0.0, seed=0, **kw):
    a = a.astype(dt)
    A = _mat(a, **kw)
    rng = np.random.default_rng(seed)
    x = rng.uniform(-1, 1, a.ncols).astype(dt)
    y0 = rng.uniform(-1, 1, a.nrows).astype(dt) if beta != 0 else None
    y = _run(torch, A, x, alpha, beta, y0, a.nrows)
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x, alpha, beta, y0)
    err = coo.parity_error(y, yref, scale)
    assert err <= TOL[dt], f"parity error {err:.3e}"
    return A, err


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("dt", [np.float64, np.float32])
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (-0.75, 0.0), (1.0, 1.0), (-0.75, 0.5)])
def test_c1_parity(torch_cuda, dt, alpha, beta, variant):
    A, _ = _parity(torch_cuda, gen.config1(), dt, alpha, beta, variant=variant)
    assert A.info()["variant"] == variant


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_c2_reduced_parity(torch_cuda, dt, variant):
    _parity(torch_cuda, gen.config2(n=40), dt, -0.75, 0.5, variant=variant)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_c3_reduced_parity(torch_cuda, dt, variant):
    A, _ = _parity(torch_cuda, gen.config3(n=36), dt, 1.0, 0.0, variant=variant)
    assert A.info()["nscatter"] > 0


@pytest.mark.parametrize("variant", VARIANTS)
def test_c4_reduced_parity(torch_cuda, variant):
    _parity(torch_cuda, gen.config4(n=300_000), np.float32, 1.0, 0.0, variant=variant)


@pytest.mark.parametrize("dt,alpha,beta", [(np.float32, 1.0, 0.0), (np.float64, -0.75, 0.5)])
def test_jit_occupancy_ranges(torch_cuda, dt, alpha, beta):
    """C4's four row-range patterns (19 / 11 / 9 / 9 diagonals) need 4, 7 and
    8 CTAs-per-SM staging sizes: the one-GPU JIT launch is split into one
    launch per occupancy class (jit_plan_ranges), each with its own dynamic
    shared memory. Every range must reproduce the oracle, with alpha/beta;
    CRSD_TUNE_JIT_ONE_LAUNCH (one launch) and CRSD_TUNE_JIT_SEQUENTIAL (the
    ranges one after another) must give the same bits."""
    from paper_conf_icpp_sunzwzyr11_b200 import TUNE_JIT_ONE_LAUNCH, TUNE_JIT_SEQUENTIAL

    # 8M rows: long enough that the split pays under jit_plan_ranges' rule
    # (the gain grows with the rows, the boundary cost is one wave)
    a = gen.config4(n=8_000_000)
    A, _ = _parity(torch_cuda, a, dt, alpha, beta, variant=4, mrows=512)
    assert A.last_launch_count() > 1
    rng = np.random.default_rng(0)
    x = rng.uniform(-1, 1, a.ncols).astype(dt)
    y0 = rng.uniform(-1, 1, a.nrows).astype(dt)
    y1 = _run(torch_cuda, A, x, alpha, beta, y0, a.nrows)
    B = _mat(a.astype(dt), variant=4, mrows=512, tune=TUNE_JIT_ONE_LAUNCH)
    y2 = _run(torch_cuda, B, x, alpha, beta, y0, a.nrows)
    assert B.last_launch_count() == 1
    assert np.array_equal(y1, y2)
    C = _mat(a.astype(dt), variant=4, mrows=512, tune=TUNE_JIT_SEQUENTIAL)
    y3 = _run(torch_cuda, C, x, alpha, beta, y0, a.nrows)
    assert C.last_launch_count() > 1
    assert np.array_equal(y1, y3)
    # range handles keep their concurrent launches (no PDL chain)
    assert A.info()["pdl"] == 0 and A.info()["jit_launches"] == A.last_launch_count()
    assert B.info()["pdl"] == 1 and B.info()["jit_launches"] == 1


@pytest.mark.parametrize("flag", ["NO_SLAB", "NO_PDL", "NO_REGSTAGE"])
@pytest.mark.parametrize("case", ["c1:f64", "c3s:f64", "c3:f64", "c3:f32", "c2s:f64", "c4:f32", "rand:f64", "rand:f32", "dense:f64"])
def test_jit_schedule_flags_full(torch_cuda, case, flag):
    """The kept scheduling alternatives at full size (CRSD_TUNE_JIT_NO_SLAB:
    scatter points through the segment descriptor; CRSD_TUNE_JIT_NO_PDL:
    plain launches): every segment once (y NaN-filled, beta = 0; then
    alpha/beta back to back), the same bits as the default codelets, and the
    oracle on sampled rows."""
    import paper_conf_icpp_sunzwzyr11_b200 as P

    torch = torch_cuda
    cfg, dts = case.split(":")
    dt = np.float64 if dts == "f64" else np.float32
    a = {"c1": lambda: gen.config1(), "c3s": lambda: gen.config3(n=96), "c3": lambda: cached("c3", gen.config3, n=192),
         "c2s": lambda: gen.config2(n=128), "c4": lambda: gen.config4(n=8_000_000),
         "rand": lambda: gen.random_diagonal(40000, 39000, 7, ndiag=12, max_off=900, p_break=0.02, max_break=400, n_scatter=2000),
         "dense": lambda: gen.random_diagonal(8192, 8192, 5, ndiag=3, n_scatter=30000, max_off=64)}[cfg]().astype(dt)
    tdt = torch.float64 if dt == np.float64 else torch.float32
    rng = np.random.default_rng(13)
    x = rng.uniform(-1, 1, a.ncols).astype(dt)
    y0 = rng.uniform(-1, 1, a.nrows).astype(dt)
    xd = torch.from_numpy(x).cuda()
    outs = []
    for tune in (0, getattr(P, "TUNE_JIT_" + flag)):
        A = _mat(a, variant=4, mrows=512 if cfg == "c4" else 0, tune=tune)
        if case == "c3:f64" and flag == "NO_REGSTAGE":
            # the north-star matrix runs register-staged as one launch by
            # default, as 5 occupancy-class ranges without
            inf = A.info()
            assert (inf["regstage"], inf["jit_launches"]) == ((1, 1) if tune == 0 else (0, 5))
        y = torch.full((a.nrows,), float("nan"), dtype=tdt, device="cuda")
        A.spmv(xd, y, 1.0, 0.0)
        y2 = torch.from_numpy(y0).cuda()
        for _ in range(3):  # back to back; the last one counts
            y2.copy_(torch.from_numpy(y0).cuda())
            A.spmv(xd, y2, -0.75, 0.5)
        torch.cuda.synchronize()
        outs.append((y.cpu().numpy(), y2.cpu().numpy()))
        A.close()
    assert not np.isnan(outs[1][0]).any()
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])
    rows = np.unique(np.concatenate([np.arange(0, a.nrows, max(1, a.nrows // 20000)), [a.nrows - 1]]))
    o = np.lexsort((a.col, a.row))
    ptr = np.searchsorted(a.row[o], np.arange(a.nrows + 1))
    yref, scale = coo.rows_spmv(rows, ptr, a.col[o], a.val[o], x, -0.75, 0.5, y0)
    assert coo.parity_error(outs[1][1][rows], yref, scale) <= TOL[dt]


@pytest.mark.parametrize("case", ["c3:f64", "c3:f32", "c2:f64", "c4:f32"])
def test_pdl_dependent_chain(torch_cuda, case):
    """Programmatic dependent launch (the default for one-launch handles;
    CRSD_TUNE_JIT_NO_PDL turns it off) lets each SpMV start while the
    previous kernel drains: its CTAs stream the matrix values first and wait
    (griddepcontrol.wait) before touching x or y. A ping-pong chain
    u_{k+1} = alpha A u_k + beta u_{k-1}, issued back to back with no host
    sync, has both hazards PDL must respect -- step k+1 reads what step k
    writes (RAW) and writes what step k reads (WAR). It must give the bits of
    the plain launches, and its first step the oracle's. C4 (occupancy-class
    ranges) stays on plain concurrent launches."""
    from paper_conf_icpp_sunzwzyr11_b200 import TUNE_JIT_NO_PDL

    torch = torch_cuda
    cfg, dts = case.split(":")
    dt = np.float64 if dts == "f64" else np.float32
    a = {"c3": lambda: gen.config3(n=96), "c2": lambda: gen.config2(n=128), "c4": lambda: gen.config4(n=8_000_000)}[cfg]()
    a = a.astype(dt)
    tdt = torch.float64 if dt == np.float64 else torch.float32
    rng = np.random.default_rng(11)
    v0 = rng.uniform(-1, 1, a.nrows).astype(dt)
    v1 = rng.uniform(-1, 1, a.nrows).astype(dt)
    alpha, beta = 0.03, 0.5
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, v1, alpha, beta, v0)
    outs = []
    for tune in (TUNE_JIT_NO_PDL, 0):
        A = _mat(a, variant=4, mrows=512 if cfg == "c4" else 0, tune=tune)
        inf = A.info()
        assert inf["pdl"] == (1 if tune == 0 and inf["jit_launches"] == 1 else 0)
        assert inf["jit_launches"] == 1 or cfg in ("c3", "c4")
        # b = [u_{k-1}, u_k]; step k: b[k % 2] <- alpha A b[(k + 1) % 2] + beta b[k % 2]
        b = [torch.from_numpy(v0).cuda(), torch.from_numpy(v1).cuda()]
        A.spmv(b[1], b[0], alpha, beta)
        torch.cuda.synchronize()
        first = b[0].cpu().numpy().copy()
        for k in range(1, 24):
            A.spmv(b[(k + 1) % 2], b[k % 2], alpha, beta)
        torch.cuda.synchronize()
        outs.append((first, [u.cpu().numpy().copy() for u in b]))
        A.close()
    assert coo.parity_error(outs[0][0], yref, scale) <= TOL[dt]
    assert np.array_equal(outs[0][0], outs[1][0])
    for u, w in zip(outs[0][1], outs[1][1]):
        assert np.array_equal(u, w)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_random_diagonal_parity(torch_cuda, seed, dt, variant):
    """Random offsets (AD runs), breaks, scatter, rectangular shapes, ragged tails."""
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 5000))
    m = int(rng.integers(1, 5000))
    a = gen.random_diagonal(n, m, seed, ndiag=int(rng.integers(1, 30)), max_off=int(rng.integers(1, 3000)), p_break=0.02, max_break=400, n_scatter=int(rng.integers(0, 300)))
    mrows = [64, 256, 512][seed % 3] if dt == np.float64 else [128, 512, 1024 if variant != 3 else 384][seed % 3]
    _parity(torch_cuda, a, dt, [1.0, -0.75][seed % 2], [0.0, 0.5][(seed // 2) % 2], seed=seed, mrows=mrows, variant=variant)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_dense_scatter_segments(torch_cuda, dt, variant):
    """Segments with hundreds of scatter points (binary-search path of the scatter pass)."""
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDError

    n = 2048
    a = gen.random_diagonal(n, n, 5, ndiag=3, n_scatter=3000)
    try:
        A, _ = _parity(torch_cuda, a, dt, 1.0, 0.0, variant=variant)
    except CRSDError as e:
        # the staged x windows of its many far-apart diagonals exceed shared
        # memory: the staged variants must refuse, AUTO must pick one that fits
        assert variant in (2, 3, 4) and "UNSUPPORTED" in str(e)
        A, _ = _parity(torch_cuda, a, dt, 1.0, 0.0, variant=0)
        assert A.info()["variant"] != variant
    P = A.export()
    assert A.info()["nscatter"] > 1000 and np.max(np.diff(P["scat_ptr"])) > 32


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("idle_max", [1, 8, 63])
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_idle_max_sweep_device(torch_cuda, dt, idle_max, variant):
    """The idle threshold decides which gaps are bridged by fills
    and which nonzeros fall to the scatter list. On the device path the built
    layout must equal the oracle's paper-order build for every threshold, and
    every kernel variant must stay within tolerance of the definition."""
    from oracle import crsd_ref
    from tests.test_builder import assert_layout_equal

    a = gen.random_diagonal(3000, 3100, 11 + idle_max, ndiag=9, max_off=700, p_break=0.05,
                            max_break=80, n_scatter=150).astype(dt)
    A, _ = _parity(torch_cuda, a, dt, -0.75, 0.5, seed=idle_max, mrows=128, idle_max=idle_max, variant=variant)
    R = crsd_ref.build(a.nrows, a.ncols, a.row, a.col, a.val, mrows=128, idle_max=idle_max, dtype=dt)
    assert_layout_equal(A.export(), crsd_ref.to_layout(R))


def test_beta_zero_never_reads_y(torch_cuda):
    a = gen.config1()
    A = _mat(a)
    x = np.random.default_rng(1).uniform(-1, 1, a.ncols)
    y = _run(torch_cuda, A, x, 1.0, 0.0, None, a.nrows)  # y prefilled with NaN
    assert np.all(np.isfinite(y))


def test_tiny_and_empty(torch_cuda):
    e = np.empty(0, np.int64)
    A = gen.COO(5, 7, e, e.copy(), np.empty(0))
    _parity(torch_cuda, A, np.float64, 1.0, 0.5)
    one = gen.COO(1, 1, np.array([0]), np.array([0]), np.array([2.5]))
    _parity(torch_cuda, one, np.float64, 1.0, 0.0)
    _parity(torch_cuda, one, np.float32, 2.0, 1.0)


def test_misaligned_vectors_rejected(torch_cuda):
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDError

    torch = torch_cuda
    a = gen.config1()
    A = _mat(a)
    x = torch.zeros(a.ncols + 1, device="cuda", dtype=torch.float64)
    y = torch.zeros(a.nrows, device="cuda", dtype=torch.float64)
    with pytest.raises(CRSDError, match="INVALID_ARG"):
        A.spmv(x[1:], y)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("n", [24, 96])
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_spmv_host_e2e(torch_cuda, dt, n, variant):
    """crsd_spmv_host: chunked H2D / compute / D2H pipeline (16 chunks at n=96)."""
    a = gen.config3(n=n).astype(dt)
    A = _mat(a, variant=variant)
    rng = np.random.default_rng(3)
    x = rng.uniform(-1, 1, a.ncols).astype(dt)
    y0 = rng.uniform(-1, 1, a.nrows).astype(dt)
    y = y0.copy()
    A.spmv_host(x, y, -0.75, 0.5)
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x, -0.75, 0.5, y0)
    assert coo.parity_error(y, yref, scale) <= TOL[dt]
    y2 = np.full(a.nrows, np.nan, dt)
    A.spmv_host(x, y2, 1.0, 0.0)
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x)
    assert coo.parity_error(y2, yref, scale) <= TOL[dt]
    if n == 96:
        assert A.last_launch_count() > 8  # chunked pipeline


# ---------------------------------------------------------------- full sizes
@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("dt", [np.float64, np.float32])
@pytest.mark.parametrize("xkind", ["linear", "quadratic"])
def test_c2_full_closed_form(torch_cuda, dt, xkind, variant):
    """BASELINE config 2 at full size (256^3), every row vs the closed form (exact)."""
    dims = (256, 256, 256)
    a = cached("c2x", gen.config2, values="exact").astype(dt)
    A = _mat(a, variant=variant)
    x = gen.vectors(a.ncols, xkind, dims=dims).astype(dt)
    y = _run(torch_cuda, A, x, 1.0, 0.0, None, a.nrows)
    assert np.array_equal(y.astype(np.float64), closed_forms.stencil_apply(dims, "7pt", xkind))


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_c2_full_random_parity(torch_cuda, dt):
    """Config 2 at full size with perturbed values, every row vs the oracle."""
    _parity(torch_cuda, cached("c2", gen.config2), dt, -0.75, 0.5)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("dt", [np.float64, np.float32])
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (-0.75, 0.5)])
def test_c3_full_parity(torch_cuda, dt, variant, alpha, beta):
    """Config 3 at full size (192^3 27-pt, idle blocks, 0.1% scatter), every
    row, in the default height the bench uses (AUTO mrows: 256 for both
    precisions), with and without alpha/beta."""
    A, _ = _parity(torch_cuda, cached("c3", gen.config3), dt, alpha, beta, variant=variant)
    inf = A.info()
    assert inf["nscatter"] > 100_000 and inf["mrows"] == 256


def test_c3_full_closed_form_ones(torch_cuda):
    """C3 stencil part with center = present couplings: A*1 == sum of the row's scatter values."""
    a = cached("c3x", gen.config3, values="exact")
    A = _mat(a)
    y = _run(torch_cuda, A, np.ones(a.ncols), 1.0, 0.0, None, a.nrows)
    nsc = int(round((3 * 192 - 2) ** 3 * 0.001))
    expect = np.zeros(a.nrows)
    np.add.at(expect, a.row[-nsc:], a.val[-nsc:])
    # scatter rows sum a few U(-1,1) values: compare with the oracle tolerance
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, np.ones(a.ncols))
    assert coo.parity_error(y, yref, scale) <= 1e-12
    assert np.max(np.abs(yref - expect)) <= 1e-12


# ---------------------------------------------------------------- row-partitioned compute
@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("case", ["c2", "c3", "c4"])
@pytest.mark.parametrize("world", [2, 3])
def test_dist_compute_single_gpu(torch_cuda, case, world, variant):
    """crsd_spmv_dist with comm=NULL: P logical ranks on one GPU, halos filled
    from the global x on the host; interior + boundary lists must reproduce
    the global product rows of each rank."""
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, partition_rows

    torch = torch_cuda
    if case == "c2":
        a, dt, mrows = gen.config2(n=40), np.float64, 256
    elif case == "c3":
        a, dt, mrows = gen.config3(n=36), np.float64, 256
    else:
        a, dt, mrows = gen.config4(n=300_000), np.float32, 512
    a = a.astype(dt)
    n = a.nrows
    x = np.random.default_rng(2).uniform(-1, 1, n).astype(dt)
    yref, scale = coo.coo_spmv(n, n, a.row, a.col, a.val, x)
    bounds = partition_rows(n, mrows, world, np.bincount(a.row, minlength=n).astype(np.float64))
    tdt = torch.float64 if dt == np.float64 else torch.float32
    for r in range(world):
        rb, re = int(bounds[r]), int(bounds[r + 1])
        m = (a.row >= rb) & (a.row < re)
        A = CRSDMatrix.from_coo(n, n, a.row[m], a.col[m], a.val[m], mrows=mrows, row_range=(rb, re), variant=variant)
        inf = A.info()
        lo, nloc, hi = A.x_layout()
        xp = np.zeros(lo + nloc + hi, dt)
        hlv, hhv = inf["halo_lo_valid"], inf["halo_hi_valid"]
        xp[lo - hlv : lo + nloc + hhv] = x[rb - hlv : re + hhv]
        xd = torch.from_numpy(xp).to("cuda", tdt)
        yd = torch.full((nloc,), float("nan"), device="cuda", dtype=tdt)
        A.spmv_dist(xd, yd, 1.0, 0.0, None)
        torch.cuda.synchronize()
        err = coo.parity_error(yd.cpu().numpy(), yref[rb:re], scale[rb:re])
        assert err <= TOL[dt], (r, err)
        assert 1 <= A.last_launch_count() <= 10  # interior range (one launch per occupancy class) + boundary list


def test_nccl_comm_world1(torch_cuda):
    """The NCCL plumbing of crsd_spmv_dist on one GPU: a 1-rank torch.distributed
    (nccl) group, crsd_comm_init_rank, crsd_dist_bind (allgather of the row
    ranges) and crsd_spmv_dist with a communicator (empty halo plan)."""
    import os
    import socket

    import torch.distributed as dist

    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, Comm

    torch = torch_cuda
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK="0", WORLD_SIZE="1")
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda:0"))
    try:
        a = gen.config2(n=40)
        n = a.nrows
        A = CRSDMatrix.from_coo(n, n, a.row, a.col, a.val, row_range=(0, n), device=0)
        comm = Comm(0, 1, 0)
        A.dist_bind(comm)
        lo, nloc, hi = A.x_layout()
        assert (lo, nloc, hi) == (0, n, 0)
        x = np.random.default_rng(4).uniform(-1, 1, n)
        xd = torch.from_numpy(x).to("cuda:0")
        yd = torch.full((n,), float("nan"), device="cuda:0", dtype=torch.float64)
        A.spmv_dist(xd, yd, 1.0, 0.0, comm)
        torch.cuda.synchronize()
        yref, scale = coo.coo_spmv(n, n, a.row, a.col, a.val, x)
        assert coo.parity_error(yd.cpu().numpy(), yref, scale) <= 1e-12
        comm.close()
    finally:
        dist.destroy_process_group()


def test_p2p_comm_world1_nccl_plumbing(torch_cuda):
    """The peer-memory communicator bootstrapped over an NCCL process group
    (the plumbing bench.py uses under torchrun: handles and range table
    allgathered as CUDA tensors), one rank: empty halo plan, exchange kernels
    with no peers, allreduce of one rank, CG graph batches through it."""
    import os
    import socket

    import torch.distributed as dist

    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, P2PComm

    torch = torch_cuda
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK="0", WORLD_SIZE="1")
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda:0"))
    try:
        a = gen.config2(n=40)
        n = a.nrows
        A = CRSDMatrix.from_coo(n, n, a.row, a.col, a.val, row_range=(0, n), device=0)
        comm = P2PComm(0, 1, 0)
        A.dist_bind(comm)
        x = np.random.default_rng(4).uniform(-1, 1, n)
        xd = torch.from_numpy(x).to("cuda:0")
        yd = torch.full((n,), float("nan"), device="cuda:0", dtype=torch.float64)
        for _ in range(3):
            A.spmv_dist(xd, yd, 1.0, 0.0, comm)
        torch.cuda.synchronize()
        yref, scale = coo.coo_spmv(n, n, a.row, a.col, a.val, x)
        assert coo.parity_error(yd.cpu().numpy(), yref, scale) <= 1e-12
        v = torch.tensor([1.5, -2.0], dtype=torch.float64, device="cuda:0")
        comm.allreduce_f64(v)
        torch.cuda.synchronize()
        assert v.cpu().tolist() == [1.5, -2.0]
        assert comm.error() == 0
        comm.close()
    finally:
        dist.destroy_process_group()


def _host_ram_gb():
    try:
        import psutil

        return psutil.virtual_memory().available / 2**30
    except Exception:
        return 0.0


# full-size tests (~2 minutes together on a B200 box with 196 GB of host RAM);
# CRSD_SKIP_SLOW=1 skips them
SLOW = pytest.mark.skipif(bool(os.environ.get("CRSD_SKIP_SLOW")), reason="CRSD_SKIP_SLOW set")


@pytest.mark.slow
@SLOW
def test_c4_full_every_row(torch_cuda):
    """BASELINE config 4 at full size (100M rows, 19 offsets / 4 patterns,
    fp32) on one GPU in the AUTO variant, alpha = -0.75, beta = 0.5: EVERY
    row against the long-double definition (oracle.coo_spmv)."""
    if _host_ram_gb() < 60:
        pytest.skip("needs ~60 GB of host RAM for the 1.19e9-entry COO")
    torch = torch_cuda
    n = 100_000_000
    a = gen.config4(n=n)
    a = gen.COO(n, n, a.row, a.col, a.val.astype(np.float32))
    A = _mat(a)
    inf = A.info()
    assert inf["nnz"] == a.nnz and inf["nscatter"] == 0 and inf["variant"] == 4
    rng = np.random.default_rng(9)
    x = rng.uniform(-1, 1, n).astype(np.float32)
    y0 = rng.uniform(-1, 1, n).astype(np.float32)
    y = _run(torch, A, x, -0.75, 0.5, y0, n)
    assert A.last_launch_count() >= 1
    del A
    yref, scale = coo.coo_spmv(n, n, a.row, a.col, a.val, x, -0.75, 0.5, y0)
    err = coo.parity_error(y, yref, scale)
    assert err <= TOL[np.float32], err


@pytest.mark.slow
@SLOW
def test_c5_full_single_handle_closed_form(torch_cuda):
    """BASELINE config 5 at full size exactly as bench.py times it at N = 1:
    one handle over all 452,984,832 rows, built by crsd_create_from_csr from
    the C generator's CSR (read in place), AUTO variant. Every row of
    y = A x and of y = -0.75 A x + 0.5 y0 is compared with the closed form
    (x affine in the grid coordinates, y0 integer: every value exact)."""
    if _host_ram_gb() < 110:
        pytest.skip("needs ~110 GB of host RAM (50 GB CSR + 25 GB CRSD values + vectors)")
    import bench
    from gen import fast
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix

    torch = torch_cuda
    nn = 768
    dims = (nn, nn, nn)
    n = nn**3
    ptr, col, val = fast.stencil(dims, bench._stencil_disps("7pt", dims), False, False, 5, None, 0, n, csr=True)
    A = CRSDMatrix.from_csr(n, n, ptr, col, val, device=0)
    del ptr, col, val
    inf = A.info()
    assert inf["nnz"] == 3_167_354_880 and inf["variant"] == 4
    coef = (3.0, (1.0, -2.0, 5.0))
    xd = torch.empty(n, dtype=torch.float64, device="cuda")
    y0 = torch.empty(n, dtype=torch.float64, device="cuda")
    ch = 1 << 26
    for r0 in range(0, n, ch):
        r1 = min(n, r0 + ch)
        g = gen.matrices.grid_coords(dims, r0, r1)
        xd[r0:r1] = torch.from_numpy(coef[0] + coef[1][0] * g[0] + coef[1][1] * g[1] + coef[1][2] * g[2])
        y0[r0:r1] = torch.from_numpy((g[0] - 2 * g[1] + 3 * g[2]).astype(np.float64))
    yd = torch.full((n,), float("nan"), dtype=torch.float64, device="cuda")
    A.spmv(xd, yd, 1.0, 0.0)
    y2 = y0.clone()
    A.spmv(xd, y2, -0.75, 0.5)
    torch.cuda.synchronize()
    for r0 in range(0, n, ch):
        r1 = min(n, r0 + ch)
        ref = closed_forms.stencil_apply(dims, "7pt", "linear", coef, r0, r1)
        assert np.array_equal(yd[r0:r1].cpu().numpy(), ref), r0
        exp2 = -0.75 * ref + 0.5 * y0[r0:r1].cpu().numpy()
        assert np.array_equal(y2[r0:r1].cpu().numpy(), exp2), r0


@pytest.mark.slow
@SLOW
@pytest.mark.parametrize("rank", [0, 3])
def test_c5_rank_block_closed_form(torch_cuda, rank):
    """BASELINE config 5 (7-pt 768^3, fp64) split into 8 row blocks as the
    8-GPU run would: one rank's block is built with its global row range, its
    x halo filled from the global x, and every row of the block is compared
    with the closed form (exact integers) -- the full-size multi-GPU layout on
    one GPU, without NCCL."""
    if _host_ram_gb() < 48:
        pytest.skip("needs ~48 GB of host RAM for a 56.6M-row block")
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, partition_rows

    torch = torch_cuda
    nn = 768
    dims = (nn, nn, nn)
    n = nn**3
    bounds = partition_rows(n, 256, 8)
    rb, re = int(bounds[rank]), int(bounds[rank + 1])
    a = gen.config5(n=nn, values="exact", row_begin=rb, row_end=re)
    A = CRSDMatrix.from_coo(n, n, a.row, a.col, a.val, row_range=(rb, re))
    del a
    inf = A.info()
    lo, nloc, hi = A.x_layout()
    hlv, hhv = inf["halo_lo_valid"], inf["halo_hi_valid"]
    # halos: the +-768^2 diagonals (plus the vector-window slack of a few elements)
    assert (hlv == 0 if rank == 0 else nn * nn <= hlv <= nn * nn + 8) and nn * nn <= hhv <= nn * nn + 8
    coef = (3.0, (1.0, -2.0, 5.0))
    g = gen.matrices.grid_coords(dims, rb - hlv, re + hhv)
    xp = np.zeros(lo + nloc + hi)
    xp[lo - hlv : lo + nloc + hhv] = coef[0] + coef[1][0] * g[0] + coef[1][1] * g[1] + coef[1][2] * g[2]
    del g
    xd = torch.from_numpy(xp).to("cuda")
    del xp
    yd = torch.full((nloc,), float("nan"), device="cuda", dtype=torch.float64)
    A.spmv_dist(xd, yd, 1.0, 0.0, None)
    torch.cuda.synchronize()
    y = yd.cpu().numpy()
    ref = closed_forms.stencil_apply(dims, "7pt", "linear", coef, rb, re)
    assert np.array_equal(y, ref)


@pytest.mark.parametrize("case", ["c1", "c3s", "band"])
def test_autotune_picks_fastest_and_keeps_parity(torch_cuda, case):
    """crsd_autotune times every applicable variant and keeps the fastest;
    the tuned handle still matches the oracle."""
    a = {"c1": gen.config1, "c3s": lambda: gen.config3(n=36), "band": lambda: gen.config4(n=300_000)}[case]()
    a = a.astype(np.float64)
    A = _mat(a)
    torch = torch_cuda
    x = np.random.default_rng(3).uniform(-1, 1, a.ncols)
    xd = torch.from_numpy(x).to("cuda")
    yd = torch.empty(a.nrows, dtype=torch.float64, device="cuda")
    r = A.autotune(xd, yd, reps=5)
    ms = {v: t for v, t in r["ms"].items() if t is not None}
    assert r["chosen"] in ms and ms[r["chosen"]] == min(ms.values())
    assert A.info()["variant"] == r["chosen"]
    y = _run(torch, A, x, -0.75, 0.0, None, a.nrows)
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x, -0.75, 0.0, None)
    assert coo.parity_error(y, yref, scale) <= TOL[np.float64]


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("dt", [np.float64, np.float32])
@pytest.mark.parametrize("case", ["c1", "c3s", "rand"])
def test_paper_ell_mode(torch_cuda, case, dt, variant):
    """CRSD_PAPER_ELL (the paper's two-part kernel):
    scatter rows are overwritten by the ELL part -- bit-exact against the
    oracle's paper-order row products (separately rounded, ascending
    columns); every other row matches the definition within tolerance."""
    from paper_conf_icpp_sunzwzyr11_b200 import CRSD_PAPER_ELL, CRSDError
    from oracle import crsd_ref

    # (Fig. 2 itself needs mrows = 2, below the GPU minimum; its ELL arrays
    # are checked against Fig. 4 on the host: test_paper_ell_export_fig2_golden)
    if case == "c1":
        a = gen.config1()
    elif case == "c3s":
        a = gen.config3(n=24)
    else:
        a = gen.random_diagonal(3000, 2900, 7, ndiag=9, max_off=700, n_scatter=150)
    a = a.astype(dt)
    mrows = 64 if dt == np.float64 else 128
    A = _mat(a, flags=CRSD_PAPER_ELL, variant=variant, mrows=mrows)
    x = np.random.default_rng(21).uniform(-1, 1, a.ncols).astype(dt)
    y = _run(torch_cuda, A, x, -0.75, 0.0, None, a.nrows)
    R = crsd_ref.build(a.nrows, a.ncols, a.row, a.col, a.val, mrows=mrows)
    ell = crsd_ref.paper_ell_rows(R, x, alpha=-0.75, dtype=dt)
    assert len(ell) == R.num_scatter_rows > 0
    rows = np.array(sorted(ell), np.int64)
    assert np.array_equal(y[rows], np.array([ell[r] for r in rows], dtype=dt)), "ELL rows not bit-exact"
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x, -0.75, 0.0, None)
    assert coo.parity_error(y, yref, scale) <= TOL[dt]
    with pytest.raises(CRSDError, match="UNSUPPORTED"):
        _run(torch_cuda, A, x, 1.0, 0.5, np.zeros(a.nrows, dt), a.nrows)


@pytest.mark.slow
@SLOW
@pytest.mark.parametrize("case", ["c2", "c3"])
def test_full_size_device_roundtrip(torch_cuda, case):
    """BASELINE configs 2 and 3 at full size: the CRSD structure as it sits in
    HBM (crsd_export reads the device arrays back; the host copy of the
    values is dropped after upload) decodes to the canonical COO bit for bit
    (north star: "CRSD construction must round-trip bit-exact to COO")."""
    from oracle import decode

    a = cached(case, gen.config2 if case == "c2" else gen.config3)
    A = _mat(a)
    P = A.export()
    assert decode.roundtrip_equal(P, a.nrows, a.ncols, a.row, a.col, a.val)
    inf = A.info()
    assert inf["nnz"] == a.nnz


@pytest.mark.parametrize("dt", [np.float64, np.float32])
@pytest.mark.parametrize("case", ["c1", "c2s", "c3s", "c4s", "rand0", "rand1", "rand2", "dense_scatter"])
def test_jit_staging_chunks_and_issue(torch_cuda, case, dt):
    """The JIT codelet's staging chunks (opts.jit_chunk: one mbarrier per x
    window by default, the whole segment on one barrier, or windows split into
    runs of k diagonals) and its copy issue (baked instance lookup by default,
    CRSD_TUNE_JIT_DESC_ISSUE: after the descriptor load), the launch (PDL or
    not) and where a CTA finds its scatter points (the per-segment slab of the
    first 16 by default -- "dense_scatter" has segments with more, which take
    the descriptor path for the rest -- or the descriptor alone,
    CRSD_TUNE_JIT_NO_SLAB) change only when the FMAs start, never their
    order: every setting matches the oracle and all settings give the same
    bits."""
    from paper_conf_icpp_sunzwzyr11_b200 import TUNE_JIT_DESC_ISSUE, TUNE_JIT_NO_PDL, TUNE_JIT_NO_SLAB, TUNE_JIT_NO_REGSTAGE

    if case == "c1":
        a = gen.config1()
    elif case == "c2s":
        a = gen.config2(n=40)
    elif case == "c3s":
        a = gen.config3(n=36)
    elif case == "c4s":
        a = gen.config4(n=300_000)
    elif case == "dense_scatter":
        a = gen.random_diagonal(2048, 2048, 5, ndiag=3, n_scatter=3000, max_off=64)
    else:
        s = int(case[-1])
        a = gen.random_diagonal(4000 + 97 * s, 3900, 30 + s, ndiag=12, max_off=900, p_break=0.02, max_break=400, n_scatter=200)
    a = a.astype(dt)
    rng = np.random.default_rng(3)
    x = rng.uniform(-1, 1, a.ncols).astype(dt)
    y0 = rng.uniform(-1, 1, a.nrows).astype(dt)
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x, -0.75, 0.5, y0)
    first = None
    for chunk in (0, -1, 1, 5):
        for tune in (0, TUNE_JIT_DESC_ISSUE, TUNE_JIT_NO_PDL, TUNE_JIT_NO_SLAB, TUNE_JIT_NO_SLAB | TUNE_JIT_DESC_ISSUE,
                     TUNE_JIT_NO_REGSTAGE):
            A = _mat(a, variant=4, jit_chunk=chunk, tune=tune)
            y = _run(torch_cuda, A, x, -0.75, 0.5, y0, a.nrows)
            assert coo.parity_error(y, yref, scale) <= TOL[dt], (chunk, tune)
            if first is None:
                first = y
            assert np.array_equal(y, first), (chunk, tune)


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_create_autotuned(torch_cuda, dt):
    """crsd_create_autotuned: every valid mrows candidate is built and timed,
    invalid ones (not a multiple of 32*RPT) are skipped, the fastest handle is
    returned and matches the oracle."""
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix

    a = gen.config3(n=40).astype(dt)
    cands = (64, 128, 256, 100) if dt == np.float64 else (128, 256, 512, 100)
    A, ms = CRSDMatrix.autotuned(a.nrows, a.ncols, a.row, a.col, a.val, mrows_candidates=cands, reps=3)
    assert ms[100] is None and all(ms[m] is not None for m in cands[:3])
    assert A.info()["mrows"] == min(cands[:3], key=lambda m: ms[m])
    x = np.random.default_rng(8).uniform(-1, 1, a.ncols).astype(dt)
    y = _run(torch_cuda, A, x, 1.0, 0.0, None, a.nrows)
    yref, scale = coo.coo_spmv(a.nrows, a.ncols, a.row, a.col, a.val, x)
    assert coo.parity_error(y, yref, scale) <= TOL[dt]


def test_c_example_runs(torch_cuda):
    """The plain-C consumer of the C-ABI: CRSD build, SpMV vs the A*1 closed
    form (exact), CG to 1e-10 -- exit code 0."""
    import subprocess

    from paper_conf_icpp_sunzwzyr11_b200 import _build

    exe = _build.build_example()
    r = subprocess.run([exe, "40"], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "closed-form mismatches 0" in r.stdout
