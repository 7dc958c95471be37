"""ORACLE (test infrastructure only): ctypes wrapper of oracle/coo_spmv.c
and oracle/coo_native.c.

y = alpha*A*x + beta*y by definition (
BASELINE.json north_star alpha/beta form):
  coo_spmv / rows_spmv -- long double accumulation: the checker
  coo_spmv_native      -- the same loop in the matrix dtype, 1 or many
                          threads: the timed CPU baseline
The shared objects are compiled with gcc by ``__graft_entry__.build()`` or on
first use here.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "coo_spmv.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_SRC_NATIVE = os.path.join(_HERE, "coo_native.c")
_LIB_NATIVE = os.path.join(_HERE, "liboracle_native.so")
_lib = None
_lib_native = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-o", _LIB, _SRC, "-lm"]
        )
    if force or not os.path.exists(_LIB_NATIVE) or os.path.getmtime(_LIB_NATIVE) < os.path.getmtime(_SRC_NATIVE):
        # -O3 (vectorised loop control), no -march: the .so travels to the GPU box host
        subprocess.check_call(
            ["gcc", "-O3", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC", "-shared", "-o", _LIB_NATIVE,
             _SRC_NATIVE]
        )
    return _LIB


def _load_native():
    global _lib_native
    if _lib_native is None:
        build()
        lib = ctypes.CDLL(_LIB_NATIVE)
        p, i64 = ctypes.c_void_p, ctypes.c_int64
        lib.oracle_coo_native_f64.argtypes = [i64, i64, p, p, p, ctypes.c_double, p, ctypes.c_double, p, p, ctypes.c_int]
        lib.oracle_coo_native_f32.argtypes = [i64, i64, p, p, p, ctypes.c_float, p, ctypes.c_float, p, p, ctypes.c_int]
        lib.oracle_coo_native_f64.restype = lib.oracle_coo_native_f32.restype = ctypes.c_int
        _lib_native = lib
    return _lib_native


def coo_spmv_native(nrows, row, col, val, x, alpha=1.0, beta=0.0, y0=None, nthreads=1, out=None):
    """y = alpha*A*x + beta*y0 accumulated in val's dtype (float32/float64),
    ``nthreads`` OpenMP threads over row ranges. COO sorted by row. Returns y
    in the dtype (into ``out`` when given)."""
    lib = _load_native()
    dt = np.float32 if np.asarray(val).dtype == np.float32 else np.float64
    row = np.ascontiguousarray(row, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int64)
    val = np.ascontiguousarray(val, dtype=dt)
    x = np.ascontiguousarray(x, dtype=dt)
    y0 = np.ascontiguousarray(y0 if y0 is not None else np.zeros(0, dt), dtype=dt)
    if beta != 0 and y0.shape[0] != nrows:
        raise ValueError("beta != 0 needs y0 of length nrows")
    y = out if out is not None else np.empty(nrows, dtype=dt)
    fn = lib.oracle_coo_native_f32 if dt == np.float32 else lib.oracle_coo_native_f64
    rc = fn(nrows, row.shape[0], _ptr(row), _ptr(col), _ptr(val), alpha, _ptr(x), beta, _ptr(y0), _ptr(y), int(nthreads))
    if rc != 0:
        raise ValueError("coo_spmv_native needs a row-sorted COO")
    return y


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        p = ctypes.c_void_p
        i64 = ctypes.c_int64
        lib.oracle_coo_spmv_f64.argtypes = [i64, i64, i64, p, p, p, ctypes.c_double, p, ctypes.c_double, p, p, p]
        lib.oracle_coo_spmv_f32.argtypes = [i64, i64, i64, p, p, p, ctypes.c_float, p, ctypes.c_float, p, p, p]
        lib.oracle_rows_spmv_f64.argtypes = [i64, p, p, p, p, ctypes.c_double, p, ctypes.c_double, p, p, p]
        for f in (lib.oracle_coo_spmv_f64, lib.oracle_coo_spmv_f32, lib.oracle_rows_spmv_f64):
            f.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def coo_spmv(nrows, ncols, row, col, val, x, alpha=1.0, beta=0.0, y0=None):
    """Return (y_ref float64[nrows], scale float64[nrows]).

    ``val``/``x``/``y0`` dtype selects the precision: float32 inputs are taken
    exactly as given (BASELINE north_star fp32 criterion).
    """
    lib = _load()
    row = np.ascontiguousarray(row, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int64)
    f32 = np.asarray(val).dtype == np.float32
    dt = np.float32 if f32 else np.float64
    val = np.ascontiguousarray(val, dtype=dt)
    x = np.ascontiguousarray(x, dtype=dt)
    if x.shape[0] != ncols:
        raise ValueError("x has wrong length")
    if y0 is None:
        y0 = np.zeros(nrows, dtype=dt)
    y0 = np.ascontiguousarray(y0, dtype=dt)
    y = np.empty(nrows, dtype=np.float64)
    s = np.empty(nrows, dtype=np.float64)
    fn = lib.oracle_coo_spmv_f32 if f32 else lib.oracle_coo_spmv_f64
    rc = fn(nrows, ncols, row.shape[0], _ptr(row), _ptr(col), _ptr(val), alpha, _ptr(x), beta, _ptr(y0), _ptr(y), _ptr(s))
    if rc != 0:
        raise ValueError(f"oracle_coo_spmv failed rc={rc}")
    return y, s


def rows_spmv(rows_sel, row_ptr, col, val, x, alpha=1.0, beta=0.0, y0=None):
    """Definition evaluated for the selected rows only (fp64; CSR-sorted input)."""
    lib = _load()
    rows_sel = np.ascontiguousarray(rows_sel, dtype=np.int64)
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int64)
    val = np.ascontiguousarray(val, dtype=np.float64)
    x = np.ascontiguousarray(x, dtype=np.float64)
    if y0 is None:
        y0 = np.zeros(row_ptr.shape[0] - 1, dtype=np.float64)
    y0 = np.ascontiguousarray(y0, dtype=np.float64)
    y = np.empty(rows_sel.shape[0], dtype=np.float64)
    s = np.empty(rows_sel.shape[0], dtype=np.float64)
    lib.oracle_rows_spmv_f64(rows_sel.shape[0], _ptr(rows_sel), _ptr(row_ptr), _ptr(col), _ptr(val), alpha, _ptr(x), beta, _ptr(y0), _ptr(y), _ptr(s))
    return y, s


def parity_error(y, y_ref, scale):
    """max_r |y - y_ref| / scale[r]; rows with scale == 0 must match exactly
    (returns inf otherwise). SURVEY.md §8(c) pass criterion."""
    y = np.asarray(y, dtype=np.float64)
    d = np.abs(y - y_ref)
    z = scale == 0
    if np.any(d[z] != 0) or np.any(np.isnan(y)):
        return float("inf")
    nz = ~z
    if not nz.any():
        return 0.0
    return float(np.max(d[nz] / scale[nz]))
