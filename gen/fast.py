"""ctypes wrapper of gen/fastgen.c: the numpy generators of gen/matrices.py
(stencil, band) in C with OpenMP, bit for bit (tests/test_gen.py). Input
generation only; compiled by ``__graft_entry__.build()`` or on first use."""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "fastgen.c")
_LIB = os.path.join(_HERE, "libfastgen.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O3", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC", "-shared",
                               "-o", _LIB, _SRC])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P, I64, I32, U64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64
        lib.fg_stencil.argtypes = [I64, I64, I64, I32, P, I32, I32, U64, P, I64, I64, P, P, P, P, I32]
        lib.fg_stencil.restype = I64
        lib.fg_band.argtypes = [I64, I32, P, P, P, P, U64, I64, I64, P, P, P, P, I32]
        lib.fg_band.restype = I64
        _lib = lib
    return _lib


def _p(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def available() -> bool:
    try:
        _load()
        return True
    except Exception:
        return False


def stencil(dims, disps, present, random, seed, drop8, row_begin, row_end, nthreads=0, csr=False):
    """(row, col, val) of rows [row_begin, row_end) -- or (row_ptr, col, val)
    with csr=True, row_ptr from 0 over those rows; disps in ascending linear order."""
    lib = _load()
    n1, n2, n3 = dims
    d = np.ascontiguousarray(np.array(disps, dtype=np.int32).reshape(-1, 3))
    dr = None if drop8 is None else np.ascontiguousarray(np.array(drop8, dtype=np.int64))
    args = (n1, n2, n3, d.shape[0], _p(d), int(present), int(random), seed & 0xFFFFFFFFFFFFFFFF, _p(dr), row_begin, row_end)
    n = lib.fg_stencil(*args, None, None, None, None, nthreads)
    if n < 0:
        raise MemoryError("fg_stencil")
    col, val = np.empty(n, np.int64), np.empty(n, np.float64)
    if csr:
        ptr = np.empty(row_end - row_begin + 1, np.int64)
        lib.fg_stencil(*args, None, _p(ptr), _p(col), _p(val), nthreads)
        return ptr, col, val
    row = np.empty(n, np.int64)
    lib.fg_stencil(*args, _p(row), None, _p(col), _p(val), nthreads)
    return row, col, val


def band(n, ranges, seed, row_begin, row_end, nthreads=0, csr=False):
    """(row, col, val) -- or (row_ptr, col, val) with csr=True -- of rows [row_begin, row_end)."""
    lib = _load()
    ra = np.array([r[0] for r in ranges], np.int64)
    rb = np.array([r[1] for r in ranges], np.int64)
    offs = [np.array(sorted(r[2]), np.int64) for r in ranges]
    optr = np.zeros(len(ranges) + 1, np.int64)
    optr[1:] = np.cumsum([o.shape[0] for o in offs])
    oc = np.ascontiguousarray(np.concatenate(offs) if offs else np.zeros(0, np.int64))
    args = (n, len(ranges), _p(ra), _p(rb), _p(optr), _p(oc), seed & 0xFFFFFFFFFFFFFFFF, row_begin, row_end)
    m = lib.fg_band(*args, None, None, None, None, nthreads)
    if m < 0:
        raise MemoryError("fg_band")
    col, val = np.empty(m, np.int64), np.empty(m, np.float64)
    if csr:
        ptr = np.empty(row_end - row_begin + 1, np.int64)
        lib.fg_band(*args, None, _p(ptr), _p(col), _p(val), nthreads)
        return ptr, col, val
    row = np.empty(m, np.int64)
    lib.fg_band(*args, _p(row), None, _p(col), _p(val), nthreads)
    return row, col, val
