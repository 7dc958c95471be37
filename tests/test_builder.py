"""Host CRSD builder (libcrsd, C++) against the oracle (CPU only).

Integer/index work is compared bit-exactly: the product's export must equal
the paper-order construction of oracle.crsd_ref (instances, offsets, value
array bytes, scatter lists), and must round-trip to the canonical COO through
the independent oracle decoder.
"""
import ctypes
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import gen
from oracle import crsd_ref, decode
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, CRSDError, CRSD_SUM_DUPLICATES, CRSD_DROP_ZEROS
from paper_conf_icpp_sunzwzyr11_b200 import crsd as C
from tests.conftest import fig2_value


def _bits(a):
    a = np.ascontiguousarray(a)
    return a.view(np.uint64 if a.dtype == np.float64 else np.uint32)


def assert_layout_equal(P, L):
    assert P["inst_first_seg"].tolist() == L["inst_first_seg"].tolist()
    assert P["inst_nseg"].tolist() == L["inst_nseg"].tolist()
    assert P["inst_offsets"] == L["inst_offsets"]
    assert P["vals"].dtype == L["vals"].dtype
    assert np.array_equal(_bits(P["vals"]), _bits(L["vals"]))
    assert P["scat_ptr"].tolist() == L["scat_ptr"].tolist()
    assert P["scat_row"].tolist() == L["scat_row"].tolist()
    assert P["scat_col"].tolist() == L["scat_col"].tolist()
    assert np.array_equal(_bits(P["scat_val"]), _bits(L["scat_val"]))


def test_library_exports_every_header_symbol():
    import re, os

    hdr = open(os.path.join(os.path.dirname(__file__), "..", "include", "crsd.h")).read()
    declared = set(re.findall(r"\b(crsd_[a-z_0-9]+)\s*\(", hdr))
    assert declared == set(C.EXPORTED)
    lib = ctypes.CDLL(C.LIB_PATH)
    for name in declared:
        assert hasattr(lib, name), name


def test_fig2_export_equals_paper(fig2, fig2_expected):
    n, m, r, c, v, _ = fig2
    A = CRSDMatrix.from_coo(n, m, r, c, v, mrows=2, idle_max=1, host_only=True)
    P = A.export()
    R = crsd_ref.build(n, m, r, c, v, mrows=2, idle_max=1)
    assert_layout_equal(P, crsd_ref.to_layout(R))
    inf = A.info()
    assert (inf["ninst"], inf["nfills"], inf["nscatter"]) == (2, 1, 1)


@settings(max_examples=60, deadline=None)
@given(
    n=st.integers(1, 70),
    m=st.integers(1, 70),
    seed=st.integers(0, 100_000),
    mrows=st.sampled_from([1, 2, 3, 4, 7, 32]),
    im=st.integers(-1, 9),
    nz=st.integers(0, 3),
    dt=st.sampled_from([np.float64, np.float32]),
    shuffle=st.booleans(),
)
def test_builder_matches_oracle_random(n, m, seed, mrows, im, nz, dt, shuffle):
    a = gen.random_diagonal(n, m, seed, ndiag=6, p_break=0.12, max_break=6, n_scatter=5, n_zeros=nz).astype(dt)
    if shuffle:
        a = a.shuffled(seed)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=mrows, idle_max=im, host_only=True)
    P = A.export()
    R = crsd_ref.build(a.nrows, a.ncols, a.row, a.col, a.val, mrows=mrows, idle_max=im, dtype=dt)
    assert_layout_equal(P, crsd_ref.to_layout(R))
    decode.check_invariants(P, R.idle_max, a.nrows, a.ncols, a.row, a.col, a.val)


@pytest.mark.parametrize("mrows", [64, 256])
def test_builder_c1_matches_oracle(mrows):
    a = gen.config1()
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=mrows, host_only=True)
    R = crsd_ref.build(a.nrows, a.ncols, a.row, a.col, a.val, mrows=mrows)
    assert_layout_equal(A.export(), crsd_ref.to_layout(R))
    assert A.info()["nscatter"] == 16


def test_builder_reduced_c3_matches_oracle():
    a = gen.config3(n=16, scatter_frac=0.002)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=64, host_only=True)
    R = crsd_ref.build(a.nrows, a.ncols, a.row, a.col, a.val, mrows=64)
    assert_layout_equal(A.export(), crsd_ref.to_layout(R))


def test_builder_reduced_c4_structure():
    """C4 scaled to 400k rows: 4 pattern row ranges; the generator's edge rows
    drop out-of-range offsets so more instances appear near the ends."""
    a = gen.config4(n=400_000)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=512, host_only=True)
    P = A.export()
    decode.check_invariants(P, 511, a.nrows, a.ncols, a.row, a.col, a.val, check_rule=False)
    sets = [tuple(o) for o in P["inst_offsets"]]
    for _, _, offs in gen.matrices.c4_ranges(400_000):
        assert tuple(offs) in sets
    assert A.info()["nscatter"] == 0


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_roundtrip_c2_reduced(dt):
    a = gen.config2(n=48).astype(dt)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True)
    P = A.export()
    assert decode.roundtrip_equal(P, a.nrows, a.ncols, a.row, a.col, a.val)
    inf = A.info()
    assert inf["nnz"] == a.nnz and inf["nscatter"] == 0


def test_roundtrip_c3_reduced_shuffled():
    a = gen.config3(n=32).shuffled(9)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=256, host_only=True)
    P = A.export()
    decode.check_invariants(P, 255, a.nrows, a.ncols, a.row, a.col, a.val, check_rule=False)


def test_duplicates_rejected_or_summed():
    r = np.array([0, 1, 1, 1])
    c = np.array([0, 1, 1, 2])
    v = np.array([1.0, 2.0, 3.0, 4.0])
    with pytest.raises(CRSDError, match="DUPLICATE"):
        CRSDMatrix.from_coo(3, 3, r, c, v, mrows=2, host_only=True)
    A = CRSDMatrix.from_coo(3, 3, r, c, v, mrows=2, host_only=True, flags=CRSD_SUM_DUPLICATES)
    assert A.info()["nnz"] == 3
    rr, cc, vv = decode.decode(A.export())
    assert vv.tolist() == [1.0, 5.0, 4.0]


def test_index_range_rejected():
    with pytest.raises(CRSDError, match="INDEX_RANGE"):
        CRSDMatrix.from_coo(3, 3, np.array([0]), np.array([3]), np.array([1.0]), host_only=True)
    with pytest.raises(CRSDError, match="INVALID_ARG"):
        CRSDMatrix.from_coo(0, 3, np.array([], np.int64), np.array([], np.int64), np.array([]), host_only=True)


def test_explicit_zeros_kept_or_dropped():
    r = np.array([0, 1, 2, 3])
    c = np.array([0, 1, 2, 3])
    v = np.array([1.0, -0.0, 2.0, 3.0])
    A = CRSDMatrix.from_coo(4, 4, r, c, v, mrows=4, host_only=True)
    P = A.export()
    assert decode.roundtrip_equal(P, 4, 4, r, c, v)
    assert P["scat_val"].tolist() == [0.0] and np.signbit(P["scat_val"][0])
    A = CRSDMatrix.from_coo(4, 4, r, c, v, mrows=4, host_only=True, flags=CRSD_DROP_ZEROS)
    assert A.info()["nscatter"] == 0 and A.info()["nnz"] == 3


def test_empty_matrix_and_empty_segments():
    A = CRSDMatrix.from_coo(10, 10, np.array([], np.int64), np.array([], np.int64), np.array([]), mrows=4, host_only=True)
    inf = A.info()
    assert inf["nseg"] == 3 and inf["ninst"] == 1 and inf["nslots"] == 0
    P = A.export()
    assert P["inst_offsets"] == [[]]


def test_csr_input_equals_coo():
    a = gen.config1().sorted()
    ptr = np.zeros(a.nrows + 1, np.int64)
    np.add.at(ptr, a.row + 1, 1)
    ptr = np.cumsum(ptr)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=128, host_only=True)
    B = CRSDMatrix.from_csr(a.nrows, a.ncols, ptr, a.col, a.val, mrows=128, host_only=True)
    assert_layout_equal(A.export(), B.export())


@pytest.mark.parametrize("mode", ["canonical", "unsorted_cols", "duplicates", "out_of_range", "row_range"])
def test_csr_input_paths(mode):
    """crsd_create_from_csr reads canonical CSR in place (no copy of the
    entries); anything else goes through the COO canonicalisation. Both give
    the COO build's layout, and the errors of the COO path."""
    a = gen.random_diagonal(3000, 3000, 4, ndiag=9, max_off=500, n_scatter=40).sorted()
    n = a.nrows
    rb, re = (1024, 2560) if mode == "row_range" else (0, n)
    m = (a.row >= rb) & (a.row < re)
    r, c, v = a.row[m], a.col[m].copy(), a.val[m].copy()
    ptr = np.zeros(re - rb + 1, np.int64)
    ptr[1:] = np.cumsum(np.bincount(r - rb, minlength=re - rb))
    A = CRSDMatrix.from_coo(n, n, r, c, v, mrows=128, host_only=True, row_range=(rb, re))
    if mode == "unsorted_cols":
        for q in range(0, re - rb, 7):  # reverse the columns of every 7th row
            c[ptr[q]:ptr[q + 1]] = c[ptr[q]:ptr[q + 1]][::-1].copy()
            v[ptr[q]:ptr[q + 1]] = v[ptr[q]:ptr[q + 1]][::-1].copy()
    if mode == "duplicates":
        q = int(np.argmax(np.diff(ptr) >= 2))
        c[ptr[q] + 1] = c[ptr[q]]
        with pytest.raises(CRSDError, match="DUPLICATE"):
            CRSDMatrix.from_csr(n, n, ptr, c, v, mrows=128, host_only=True)
        return
    if mode == "out_of_range":
        c[5] = n + 3
        with pytest.raises(CRSDError, match="INDEX_RANGE"):
            CRSDMatrix.from_csr(n, n, ptr, c, v, mrows=128, host_only=True)
        return
    B = CRSDMatrix.from_csr(n, n, ptr, c, v, mrows=128, host_only=True, row_range=(rb, re))
    assert_layout_equal(A.export(), B.export())


def test_gpu_handle_needs_aligned_mrows():
    a = gen.config1()
    with pytest.raises(CRSDError, match="UNSUPPORTED"):
        CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=96)


def test_unique_bytes_accounting():
    a = gen.config2(n=16)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True)
    inf = A.info()
    n = a.nrows
    assert inf["unique_bytes_beta0"] == inf["nslots"] * 8 + n * 8 + n * 8
    assert inf["unique_bytes_beta1"] == inf["unique_bytes_beta0"] + n * 8


@pytest.mark.parametrize("case", ["c1", "c2s", "c3s", "rand", "empty"])
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_jit_codelets_compile_for_sm100a(case, dt, tmp_path):
    """The JIT variant's generated per-pattern codelets (the paper's code
    generator) compile for sm_100a, with one case per
    distinct pattern and the pattern offsets baked in as literals."""
    import subprocess

    if case == "c1":
        a = gen.config1()
    elif case == "c2s":
        a = gen.config2(n=24)
    elif case == "c3s":
        a = gen.config3(n=20)
    elif case == "empty":
        # segments without any diagonal: that pattern has no offsets, so its
        # offset-table start equals the next pattern's (A11)
        a = gen.config2(n=24)
        keep = (a.row < 1024) | (a.row >= 2048)
        a = gen.COO(a.nrows, a.ncols, a.row[keep], a.col[keep], a.val[keep])
    else:
        a = gen.random_diagonal(3000, 3000, 3, ndiag=8, max_off=400, n_scatter=40)
    a = a.astype(dt)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True, variant=4)
    src = A.jit_source()
    P = A.export()
    npat = A.info()["npat"]
    # one codelet + one case per distinct pattern; the baked segment ->
    # pattern lookup has one leaf per instance (the paper's Table II rows)
    import re

    assert len(re.findall(r"__device__ __forceinline__ void codelet_\d+\(", src)) == npat
    # the register-staged kernel (crsd_jit_rs, when it is used) dispatches
    # every pattern again, some into their register-staged codelets
    n_rs = src.count("crsd_jit_rs(")
    assert src.count("case ") == npat * (1 + n_rs)
    assert len(re.findall(r"void codelet_rs_\d+\(", src)) <= npat * n_rs
    assert src.count("{ key = ") == A.info()["ninst"]
    # two entry points: the plain kernel and the boundary kernel with the
    # fused halo receive (wait on the senders' flags, proxy fence, release)
    assert 'extern "C" __global__ void __launch_bounds__(NT) crsd_jit(' in src
    assert 'extern "C" __global__ void __launch_bounds__(NT) crsd_jit_halo(' in src
    assert "fence.proxy.async.global" in src and "st.release.sys" in src
    for offs in P["inst_offsets"]:
        assert "// pattern offsets: " + " ".join(str(o) for o in offs) in src
    f = tmp_path / "k.cu"
    f.write_text(src)
    r = subprocess.run(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-std=c++17", "-c", str(f), "-o", str(tmp_path / "k.o")], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr[-2000:]
    # the cubin NVRTC builds (what the GPU runs): bulk copies + mbarriers in
    # SASS, and no per-nonzero index load on the non-edge path
    cub = tmp_path / "k.cubin"
    cub.write_bytes(A.jit_cubin())
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", str(cub)], capture_output=True, text=True).stdout
    if A.info()["max_ndias"] > 0:
        assert "UBLKCP" in sass and "SYNCS" in sass


@pytest.mark.parametrize("case", ["c3s", "empty"])
def test_jit_pdl_codelets(case):
    """Codelets for programmatic dependent launch (the default for one-launch
    handles; not with CRSD_TUNE_JIT_NO_PDL): the value copies are issued before
    griddepcontrol.wait, every x window copy after it, and the kernel lets
    its dependent launch start (griddepcontrol.launch_dependents); the cubin
    holds the SASS for both (ACQBULK, PREEXIT)."""
    import subprocess

    from paper_conf_icpp_sunzwzyr11_b200 import TUNE_JIT_NO_PDL

    a = gen.config3(n=20)
    if case == "empty":
        keep = (a.row < 1024) | (a.row >= 2048)
        a = gen.COO(a.nrows, a.ncols, a.row[keep], a.col[keep], a.val[keep])
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True, variant=4)
    src = A.jit_source()
    # once per entry kernel that crsd_spmv launches (crsd_jit, and crsd_jit_rs
    # when register staging is used)
    assert src.count("griddepcontrol.launch_dependents") == 1 + src.count("crsd_jit_rs(")
    for body in src.split("__device__ __forceinline__ void codelet_")[1:]:
        body = body.split("  T acc[Q];")[0]
        w = body.index("griddepcontrol.wait")
        # value copies (a.vals) before the wait, window copies (a.x) of the
        # non-halo path only after it
        for line in body[:w].splitlines():
            if "g2s(" in line and "a.x" in line:
                assert "if (!edge) g2s" in line  # the halo kernel's windows (after halo_wait)
        assert "a.vals" not in body[w:]
    B = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True, variant=4, tune=TUNE_JIT_NO_PDL)
    assert "griddepcontrol" not in B.jit_source()
    p = "/tmp/_crsd_pdl_%d.cubin" % os.getpid()
    with open(p, "wb") as f:
        f.write(A.jit_cubin())
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", p], capture_output=True, text=True).stdout
    os.unlink(p)
    assert "ACQBULK" in sass and "PREEXIT" in sass


def test_jit_scatter_slab_codegen():
    """Matrices with scatter points: the codelets load a CTA's first 16
    points from the per-segment slab (an address known without any load) and
    read the segment descriptor only for the points beyond them;
    CRSD_TUNE_JIT_NO_SLAB keeps the descriptor-first gather; matrices without
    scatter points have no scatter code at all."""
    from paper_conf_icpp_sunzwzyr11_b200 import TUNE_JIT_NO_SLAB

    a = gen.config3(n=20)
    src = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True, variant=4).jit_source()
    assert "a.scat_slab + s * 16" in src and "if (nscat > 16)" in src and "a.scat_rec[" not in src
    src = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True, variant=4,
                              tune=TUNE_JIT_NO_SLAB).jit_source()
    assert "a.scat_slab + s" not in src and "a.scat_rec[sbeg + lane]" in src
    b = gen.config2(n=24)
    src = CRSDMatrix.from_coo(b.nrows, b.ncols, b.row, b.col, b.val, host_only=True, variant=4).jit_source()
    assert "g_mask" not in src and "scat_slab + s" not in src


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_jit_register_staging_codegen(dt):
    """Register staging (C3's 27-diagonal patterns): each register-staged
    codelet loads the values of its last R diagonals with coalesced streaming
    loads (rv<d>[q]), bulk-copies only the first nd - R value runs, and runs
    the FMAs in the plain codelet's order with the same x operands; the
    second kernel (crsd_jit_rs) dispatches to it. CRSD_TUNE_JIT_NO_REGSTAGE
    removes both. fp32 C3 (6 CTAs/SM by shared memory, 8 by threads, no
    registers to spare at 7) gets none."""
    import re

    from paper_conf_icpp_sunzwzyr11_b200 import TUNE_JIT_NO_REGSTAGE

    a = gen.config3(n=48).astype(dt)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True, variant=4)
    src = A.jit_source()
    m, es = A.info()["mrows"], np.dtype(dt).itemsize
    B = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True, variant=4, tune=TUNE_JIT_NO_REGSTAGE)
    assert "crsd_jit_rs(" not in B.jit_source() and "codelet_rs_" not in B.jit_source()
    if dt == np.float32:
        assert "crsd_jit_rs(" not in src
        return
    assert "crsd_jit_rs(" in src
    keys = re.findall(r"void codelet_rs_(\d+)\(", src)
    assert keys
    for k in keys:
        plain = src.split("void codelet_" + k + "(")[1].split("\n}\n")[0]
        rs = src.split("void codelet_rs_" + k + "(")[1].split("\n}\n")[0]
        nd = len(re.findall(r"acc\[q\] = fma\(", plain.split("} else {")[0]))
        rv = sorted(set(int(d) for d in re.findall(r"T rv(\d+)\[Q\];", rs)))
        R = len(rv)
        assert R > 0 and rv == list(range(nd - R, nd))  # a suffix of the pattern
        for d in rv:
            assert "rv%d[q] = __ldcs(a.vals + vb + %d + t + q * NT)" % (d, d * m) in rs
        copied = sum(int(b) for b in re.findall(r"g2s\(vs \+ \d+, a\.vals \+ vb \+ \d+, (\d+)u", rs))
        assert copied == (nd - R) * m * es
        # the same FMAs in the same order: x operands equal, values from
        # shared memory for d < nd - R, from registers after
        fp = re.findall(r"acc\[q\] = fma\((.*?), (xs\[\d+ \+ r\])", plain.split("} else {")[0])
        fr = re.findall(r"acc\[q\] = fma\((.*?), (xs\[\d+ \+ r\])", rs.split("} else {")[0])
        assert len(fp) == len(fr) == nd and [x for _, x in fp] == [x for _, x in fr]
        for d, ((vp, _), (vr, _)) in enumerate(zip(fp, fr)):
            assert vr == (vp if d < nd - R else "rv%d[q]" % d)
        # x windows land after the staged values
        assert "T *xs = vs + %d;" % ((nd - R) * m) in rs


def test_paper_ell_export_fig2_golden(fig2, fig2_expected):
    """CRSD_PAPER_ELL: the product's scatter-row ELL arrays equal Fig. 4's
    (num_scatter_rows, scatter_rowno, num_scatter_width, scatter_colval,
    scatter_val)."""
    from paper_conf_icpp_sunzwzyr11_b200 import CRSD_PAPER_ELL

    n, m, r, c, v, _ = fig2
    A = CRSDMatrix.from_coo(n, m, r, c, v, mrows=2, idle_max=1, host_only=True, flags=CRSD_PAPER_ELL)
    E = A.export_paper_ell()
    g = fig2_expected
    assert E["num_scatter_rows"] == g["num_scatter_rows"]
    assert E["num_scatter_width"] == g["num_scatter_width"]
    assert E["scatter_rowno"].tolist() == g["scatter_rowno"]
    assert E["scatter_colval"].tolist() == g["scatter_colval"]
    assert E["scatter_val"].tolist() == [fig2_value(s) for s in g["scatter_val"]]


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_paper_ell_export_matches_oracle(seed):
    from paper_conf_icpp_sunzwzyr11_b200 import CRSD_PAPER_ELL

    a = gen.random_diagonal(500, 460, seed, ndiag=7, n_scatter=60, n_zeros=5)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=64, host_only=True, flags=CRSD_PAPER_ELL)
    R = crsd_ref.build(a.nrows, a.ncols, a.row, a.col, a.val, mrows=64)
    E = A.export_paper_ell()
    assert E["num_scatter_rows"] == R.num_scatter_rows and E["num_scatter_width"] == R.num_scatter_width
    assert E["scatter_rowno"].tolist() == R.scatter_rowno
    assert E["scatter_colval"].tolist() == R.scatter_colval
    assert np.array_equal(_bits(E["scatter_val"]), _bits(np.array(R.scatter_val, np.float64)))


def test_paper_ell_needs_flag():
    a = gen.config1()
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True)
    with pytest.raises(Exception, match="UNSUPPORTED"):
        A.export_paper_ell()


def test_c_example_links_against_the_c_abi():
    """examples/crsd_example.c (plain C, no Python) compiles and links against
    libcrsd.so through include/crsd.h alone; it runs on the GPU in
    tests/test_gpu_spmv.py::test_c_example_runs."""
    import os
    import subprocess

    from paper_conf_icpp_sunzwzyr11_b200 import _build

    exe = _build.build_example()
    assert os.access(exe, os.X_OK)
    out = subprocess.run(["ldd", exe], capture_output=True, text=True).stdout
    assert "libcrsd.so" in out and "not found" not in out
