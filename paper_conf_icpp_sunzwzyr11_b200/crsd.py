"""Thin ctypes binding of libcrsd.so (include/crsd.h). Argument marshalling
only: every step of the SpMV runs in the library's CUDA kernels; torch is used
for device memory and streams. There is no fallback: if the library is
missing, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libcrsd.so")

CRSD_OK = 0
STATUS = {
    0: "CRSD_OK",
    1: "CRSD_ERR_INVALID_ARG",
    2: "CRSD_ERR_INDEX_RANGE",
    3: "CRSD_ERR_DUPLICATE",
    4: "CRSD_ERR_UNSUPPORTED",
    5: "CRSD_ERR_ALLOC",
    6: "CRSD_ERR_CUDA",
    7: "CRSD_ERR_NCCL",
}
CRSD_R32F, CRSD_R64F = 0, 1
CRSD_SUM_DUPLICATES, CRSD_HOST_ONLY, CRSD_DROP_ZEROS, CRSD_PAPER_ELL = 0x1, 0x2, 0x4, 0x8
VARIANT_AUTO, VARIANT_LDG, VARIANT_TMA, VARIANT_PIPE, VARIANT_JIT = 0, 1, 2, 3, 4
# opts.tune (include/crsd.h CRSD_TUNE_*)
TUNE_JIT_DESC_ISSUE, TUNE_JIT_ONE_LAUNCH, TUNE_JIT_SPLIT_ALL = 0x1, 0x2, 0x4
TUNE_JIT_SEQUENTIAL, TUNE_DIST_BOUNDARY_SERIAL, TUNE_NO_JIT = 0x8, 0x10, 0x20
TUNE_HALO_UNFUSED, TUNE_JIT_NO_PDL, TUNE_JIT_NO_SLAB, TUNE_JIT_NO_REGSTAGE = 0x40, 0x80, 0x100, 0x200

# every symbol include/crsd.h declares
EXPORTED = [
    "crsd_last_error",
    "crsd_version",
    "crsd_opts_init",
    "crsd_create_from_coo",
    "crsd_create_from_csr",
    "crsd_destroy",
    "crsd_spmv",
    "crsd_spmv_host",
    "crsd_dist_x_layout",
    "crsd_comm_unique_id",
    "crsd_comm_init_rank",
    "crsd_comm_destroy",
    "crsd_dist_bind",
    "crsd_spmv_dist",
    "crsd_dist_plan",
    "crsd_partition_rows",
    "crsd_get_info",
    "crsd_export",
    "crsd_last_launch_count",
    "crsd_jit_source",
    "crsd_jit_cubin",
    "crsd_cg",
    "crsd_autotune",
    "crsd_export_paper_ell",
    "crsd_create_autotuned",
    "crsd_comm_init_p2p",
    "crsd_comm_p2p_open",
    "crsd_dist_bind_ranges",
    "crsd_comm_allreduce_f64",
    "crsd_comm_error",
    "crsd_dist_ranges",
    "crsd_dist_x_alloc",
]


class CRSDError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class Opts(ctypes.Structure):
    _fields_ = [
        ("mrows", ctypes.c_int32),
        ("idle_max", ctypes.c_int32),
        ("flags", ctypes.c_uint32),
        ("device", ctypes.c_int32),
        ("row_begin", ctypes.c_int64),
        ("row_end", ctypes.c_int64),
        ("nthreads", ctypes.c_int32),
        ("variant", ctypes.c_int32),
        ("jit_chunk", ctypes.c_int32),
        ("tune", ctypes.c_uint32),
        ("e2e_chunks", ctypes.c_int32),
        ("reserved", ctypes.c_int32),
    ]


_INFO_FIELDS = [
    ("nrows", ctypes.c_int64), ("ncols", ctypes.c_int64),
    ("row_begin", ctypes.c_int64), ("row_end", ctypes.c_int64),
    ("mrows", ctypes.c_int32), ("idle_max", ctypes.c_int32),
    ("dtype", ctypes.c_int32), ("rows_per_thread", ctypes.c_int32),
    ("nnz", ctypes.c_int64), ("nseg", ctypes.c_int64), ("ninst", ctypes.c_int64),
    ("npat", ctypes.c_int64), ("noffsets", ctypes.c_int64), ("max_ndias", ctypes.c_int64),
    ("nslots", ctypes.c_int64), ("ndiag_nnz", ctypes.c_int64), ("nfills", ctypes.c_int64),
    ("nscatter", ctypes.c_int64), ("nedge_seg", ctypes.c_int64),
    ("halo_lo", ctypes.c_int64), ("halo_hi", ctypes.c_int64),
    ("halo_lo_valid", ctypes.c_int64), ("halo_hi_valid", ctypes.c_int64),
    ("device_bytes", ctypes.c_int64),
    ("variant", ctypes.c_int32), ("smem_bytes", ctypes.c_int32),
    ("unique_bytes_beta0", ctypes.c_int64), ("unique_bytes_beta1", ctypes.c_int64),
    ("jit_launches", ctypes.c_int32), ("pdl", ctypes.c_int32),
    ("regstage", ctypes.c_int32), ("reserved_", ctypes.c_int32),
]


class Info(ctypes.Structure):
    _fields_ = _INFO_FIELDS


class Export(ctypes.Structure):
    _fields_ = [
        ("inst_first_seg", ctypes.c_void_p),
        ("inst_nseg", ctypes.c_void_p),
        ("inst_pattern", ctypes.c_void_p),
        ("pat_ptr", ctypes.c_void_p),
        ("pat_offsets", ctypes.c_void_p),
        ("vals", ctypes.c_void_p),
        ("scat_ptr", ctypes.c_void_p),
        ("scat_row", ctypes.c_void_p),
        ("scat_col", ctypes.c_void_p),
        ("scat_val", ctypes.c_void_p),
    ]


class CGResult(ctypes.Structure):
    _fields_ = [
        ("iterations", ctypes.c_int32),
        ("converged", ctypes.c_int32),
        ("rr0", ctypes.c_double),
        ("rr", ctypes.c_double),
        ("bb", ctypes.c_double),
        ("launches", ctypes.c_int64),
    ]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is not built; run `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(LIB_PATH)
    P, I64, I32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
    sig = {
        "crsd_last_error": ([], ctypes.c_char_p),
        "crsd_version": ([], ctypes.c_char_p),
        "crsd_opts_init": ([P], ctypes.c_int),
        "crsd_create_from_coo": ([I64, I64, I64, P, P, P, ctypes.c_int, P, P], ctypes.c_int),
        "crsd_create_from_csr": ([I64, I64, P, P, P, ctypes.c_int, P, P], ctypes.c_int),
        "crsd_destroy": ([P], ctypes.c_int),
        "crsd_spmv": ([P, P, P, P, P, P], ctypes.c_int),
        "crsd_spmv_host": ([P, P, P, P, P, P], ctypes.c_int),
        "crsd_dist_x_layout": ([P, P, P, P], ctypes.c_int),
        "crsd_comm_unique_id": ([P], ctypes.c_int),
        "crsd_comm_init_rank": ([P, ctypes.c_int, ctypes.c_int, ctypes.c_int, P], ctypes.c_int),
        "crsd_comm_destroy": ([P], ctypes.c_int),
        "crsd_dist_bind": ([P, P, P], ctypes.c_int),
        "crsd_spmv_dist": ([P, P, P, P, P, P, P], ctypes.c_int),
        "crsd_dist_plan": ([ctypes.c_int, ctypes.c_int, P, P, P, P, P, P, P, P, P], ctypes.c_int),
        "crsd_partition_rows": ([I64, I32, ctypes.c_int, P, P], ctypes.c_int),
        "crsd_get_info": ([P, P], ctypes.c_int),
        "crsd_export": ([P, P], ctypes.c_int),
        "crsd_last_launch_count": ([P, P], ctypes.c_int),
        "crsd_jit_source": ([P, P, I64, P], ctypes.c_int),
        "crsd_jit_cubin": ([P, P, I64, P], ctypes.c_int),
        "crsd_cg": ([P, P, P, I32, ctypes.c_double, I32, P, P, P, P], ctypes.c_int),
        "crsd_autotune": ([P, P, P, I32, P, P, P], ctypes.c_int),
        "crsd_export_paper_ell": ([P, P, P, P, P, P], ctypes.c_int),
        "crsd_create_autotuned": ([I64, I64, I64, P, P, P, ctypes.c_int, P, P, I32, I32, P, P], ctypes.c_int),
        "crsd_comm_init_p2p": ([ctypes.c_int, ctypes.c_int, ctypes.c_int, I64, P, P], ctypes.c_int),
        "crsd_comm_p2p_open": ([P, P], ctypes.c_int),
        "crsd_dist_bind_ranges": ([P, P, P], ctypes.c_int),
        "crsd_comm_allreduce_f64": ([P, P, ctypes.c_int, P], ctypes.c_int),
        "crsd_comm_error": ([P, P], ctypes.c_int),
        "crsd_dist_ranges": ([P, P], ctypes.c_int),
        "crsd_dist_x_alloc": ([P, P, P], ctypes.c_int),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    return lib


lib = _load()


def _check(st: int):
    if st != CRSD_OK:
        raise CRSDError(st, lib.crsd_last_error().decode())


def _p(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def _dtype_code(dt) -> int:
    dt = np.dtype(dt)
    if dt == np.float64:
        return CRSD_R64F
    if dt == np.float32:
        return CRSD_R32F
    raise ValueError(f"unsupported dtype {dt}")


def _scalar(v, dt):
    return (ctypes.c_double if np.dtype(dt) == np.float64 else ctypes.c_float)(v)


def _stream_ptr(stream):
    import torch

    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


class CRSDMatrix:
    """A CRSD matrix owned by libcrsd (host structure + device arrays)."""

    def __init__(self, handle, dtype):
        self._h = ctypes.c_void_p(handle)
        self.dtype = np.dtype(dtype)

    # ------------------------------------------------------------ creation
    @classmethod
    def from_coo(
        cls,
        nrows: int,
        ncols: int,
        row,
        col,
        val,
        *,
        mrows: int = 0,
        idle_max: int = -1,
        flags: int = 0,
        host_only: bool = False,
        row_range: Optional[tuple] = None,
        device: int = -1,
        nthreads: int = 0,
        variant: int = 0,
        jit_chunk: int = 0,
        tune: int = 0,
        e2e_chunks: int = 0,
    ) -> "CRSDMatrix":
        row = np.ascontiguousarray(row, dtype=np.int64)
        col = np.ascontiguousarray(col, dtype=np.int64)
        val = np.ascontiguousarray(val)
        if val.dtype not in (np.float32, np.float64):
            val = val.astype(np.float64)
        if not (row.shape == col.shape == val.shape):
            raise ValueError("row/col/val lengths differ")
        o = Opts()
        lib.crsd_opts_init(ctypes.byref(o))
        o.mrows = mrows
        o.idle_max = idle_max
        o.flags = flags | (CRSD_HOST_ONLY if host_only else 0)
        o.device = device
        o.nthreads = nthreads
        o.variant = variant
        o.jit_chunk = jit_chunk
        o.tune = tune
        o.e2e_chunks = e2e_chunks
        if row_range is not None:
            o.row_begin, o.row_end = int(row_range[0]), int(row_range[1])
        h = ctypes.c_void_p()
        _check(
            lib.crsd_create_from_coo(
                nrows, ncols, row.shape[0], _p(row), _p(col), _p(val), _dtype_code(val.dtype), ctypes.byref(o), ctypes.byref(h)
            )
        )
        return cls(h.value, val.dtype)

    @classmethod
    def autotuned(cls, nrows, ncols, row, col, val, *, mrows_candidates=(0,), idle_max=-1, flags=0, device=-1, reps=20):
        """crsd_create_autotuned: build each mrows candidate, autotune its kernel
        variant, keep the fastest handle. Returns (matrix, {mrows: ms or None})."""
        row = np.ascontiguousarray(row, dtype=np.int64)
        col = np.ascontiguousarray(col, dtype=np.int64)
        val = np.ascontiguousarray(val)
        if val.dtype not in (np.float32, np.float64):
            val = val.astype(np.float64)
        o = Opts()
        lib.crsd_opts_init(ctypes.byref(o))
        o.idle_max, o.flags, o.device = idle_max, flags, device
        cand = np.ascontiguousarray(mrows_candidates, dtype=np.int32)
        ms = np.zeros(cand.shape[0], np.float64)
        h = ctypes.c_void_p()
        _check(
            lib.crsd_create_autotuned(
                nrows, ncols, row.shape[0], _p(row), _p(col), _p(val), _dtype_code(val.dtype), ctypes.byref(o),
                _p(cand), int(cand.shape[0]), int(reps), ctypes.byref(h), _p(ms),
            )
        )
        return cls(h.value, val.dtype), {int(m): (None if t < 0 else float(t)) for m, t in zip(cand, ms)}

    @classmethod
    def from_csr(
        cls,
        nrows,
        ncols,
        row_ptr,
        col,
        val,
        *,
        mrows=0,
        idle_max=-1,
        flags=0,
        host_only=False,
        row_range: Optional[tuple] = None,
        device=-1,
        nthreads=0,
        variant=0,
        jit_chunk=0,
        tune=0,
        e2e_chunks=0,
    ):
        """crsd_create_from_csr: row_ptr over the owned rows (row_range, default
        all rows). Canonical input (strictly increasing columns per row) is
        read in place by the builder, without a copy of the entries."""
        row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
        col = np.ascontiguousarray(col, dtype=np.int64)
        val = np.ascontiguousarray(val)
        if val.dtype not in (np.float32, np.float64):
            val = val.astype(np.float64)
        o = Opts()
        lib.crsd_opts_init(ctypes.byref(o))
        o.mrows, o.idle_max, o.flags, o.device = mrows, idle_max, flags | (CRSD_HOST_ONLY if host_only else 0), device
        o.nthreads, o.variant, o.jit_chunk, o.tune, o.e2e_chunks = nthreads, variant, jit_chunk, tune, e2e_chunks
        if row_range is not None:
            o.row_begin, o.row_end = int(row_range[0]), int(row_range[1])
        h = ctypes.c_void_p()
        _check(lib.crsd_create_from_csr(nrows, ncols, _p(row_ptr), _p(col), _p(val), _dtype_code(val.dtype), ctypes.byref(o), ctypes.byref(h)))
        return cls(h.value, val.dtype)

    def close(self):
        if self._h is not None and self._h.value:
            lib.crsd_destroy(self._h)
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ------------------------------------------------------------ compute
    def spmv(self, x, y, alpha=1.0, beta=0.0, stream=None):
        """y = alpha*A*x + beta*y with torch CUDA tensors (asynchronous)."""
        _check(
            lib.crsd_spmv(
                self._h,
                ctypes.byref(_scalar(alpha, self.dtype)),
                ctypes.c_void_p(x.data_ptr()),
                ctypes.byref(_scalar(beta, self.dtype)),
                ctypes.c_void_p(y.data_ptr()),
                _stream_ptr(stream),
            )
        )
        return y

    def spmv_host(self, x: np.ndarray, y: np.ndarray, alpha=1.0, beta=0.0, stream=None):
        """End-to-end form with host arrays (copies inside; synchronous)."""
        assert x.dtype == self.dtype and y.dtype == self.dtype and x.flags.c_contiguous and y.flags.c_contiguous
        _check(
            lib.crsd_spmv_host(
                self._h,
                ctypes.byref(_scalar(alpha, self.dtype)),
                ctypes.c_void_p(x.ctypes.data),
                ctypes.byref(_scalar(beta, self.dtype)),
                ctypes.c_void_p(y.ctypes.data),
                _stream_ptr(stream),
            )
        )
        return y

    def spmv_host_ptr(self, x_ptr: int, y_ptr: int, alpha=1.0, beta=0.0, stream=None):
        """End-to-end form with raw host pointers (e.g. pinned torch tensors)."""
        _check(
            lib.crsd_spmv_host(
                self._h,
                ctypes.byref(_scalar(alpha, self.dtype)),
                ctypes.c_void_p(x_ptr),
                ctypes.byref(_scalar(beta, self.dtype)),
                ctypes.c_void_p(y_ptr),
                _stream_ptr(stream),
            )
        )

    def spmv_dist(self, x_padded, y_local, alpha=1.0, beta=0.0, comm=None, stream=None):
        _check(
            lib.crsd_spmv_dist(
                self._h,
                ctypes.byref(_scalar(alpha, self.dtype)),
                ctypes.c_void_p(x_padded.data_ptr()),
                ctypes.byref(_scalar(beta, self.dtype)),
                ctypes.c_void_p(y_local.data_ptr()),
                comm._h if comm is not None else None,
                _stream_ptr(stream),
            )
        )
        return y_local

    def cg(self, b, x, max_iter, rtol=0.0, check_every=16, comm=None, history=False, stream=None) -> dict:
        """Conjugate gradient A x = b (crsd_cg): b, x torch CUDA tensors of the
        owned rows; x holds x0 on entry and the iterate on exit. Returns the
        crsd_cg_result_t fields (+ "rr_history" when history=True)."""
        res = CGResult()
        hist = np.zeros(max_iter + 1, np.float64) if history else None
        _check(
            lib.crsd_cg(
                self._h,
                ctypes.c_void_p(b.data_ptr()),
                ctypes.c_void_p(x.data_ptr()),
                int(max_iter),
                float(rtol),
                int(check_every),
                comm._h if comm is not None else None,
                _p(hist) if hist is not None else None,
                ctypes.byref(res),
                _stream_ptr(stream),
            )
        )
        out = {k: getattr(res, k) for k, _ in CGResult._fields_}
        if history:
            out["rr_history"] = hist[: res.iterations + 1]
        return out

    def autotune(self, x, y, reps=20, stream=None) -> dict:
        """Time every applicable kernel variant on (x, y) and keep the fastest
        (crsd_autotune). Returns {"chosen": v, "ms": {variant: ms or None}}."""
        ms = np.zeros(5, np.float64)
        ch = ctypes.c_int32()
        _check(lib.crsd_autotune(self._h, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(y.data_ptr()), int(reps), _p(ms), ctypes.byref(ch), _stream_ptr(stream)))
        return {"chosen": ch.value, "ms": {v: (None if ms[v] < 0 else float(ms[v])) for v in range(1, 5)}}

    def export_paper_ell(self) -> dict:
        """The paper's scatter-row ELL arrays of a CRSD_PAPER_ELL handle (Fig. 4 names)."""
        n, w = ctypes.c_int64(), ctypes.c_int64()
        _check(lib.crsd_export_paper_ell(self._h, ctypes.byref(n), ctypes.byref(w), None, None, None))
        rowno = np.zeros(n.value, np.int64)
        colval = np.zeros(n.value * w.value, np.int64)
        val = np.zeros(n.value * w.value, self.dtype)
        _check(lib.crsd_export_paper_ell(self._h, None, None, _p(rowno), _p(colval), _p(val)))
        return {"num_scatter_rows": n.value, "num_scatter_width": w.value, "scatter_rowno": rowno, "scatter_colval": colval, "scatter_val": val}

    def dist_bind(self, comm, stream=None, pg=None):
        """Derive the halo plan. NCCL communicators exchange the range table
        themselves (crsd_dist_bind); peer-memory ones get it allgathered here
        over torch.distributed (crsd_dist_bind_ranges)."""
        if isinstance(comm, P2PComm):
            table = comm.allgather_i64(self.dist_ranges())
            _check(lib.crsd_dist_bind_ranges(self._h, comm._h, _p(table)))
        else:
            _check(lib.crsd_dist_bind(self._h, comm._h, _stream_ptr(stream)))

    def dist_x_alloc(self, comm):
        """crsd_dist_x_alloc (collective): the library-owned padded x of this
        rank, mapped by every peer, as a CUDA tensor view (halo_lo + n_local +
        halo_hi elements; owned part at [halo_lo, halo_lo + n_local)).
        crsd_spmv_dist with it moves the halo as one-sided puts into the
        neighbours' pads. The view is valid while this handle lives."""
        import torch

        p = ctypes.c_void_p()
        _check(lib.crsd_dist_x_alloc(self._h, comm._h, ctypes.byref(p)))
        lo, n, hi = self.x_layout()

        class _View:
            __cuda_array_interface__ = {
                "shape": (lo + n + hi,),
                "typestr": "<f8" if self.dtype == np.float64 else "<f4",
                "data": (p.value, False),
                "version": 3,
            }

        t = torch.as_tensor(_View(), device=f"cuda:{torch.cuda.current_device()}")
        self._dx = t
        return t

    def dist_ranges(self) -> np.ndarray:
        """{row_begin, row_end, halo_lo_valid, halo_hi_valid} of this handle (crsd_dist_ranges)."""
        r = np.zeros(4, np.int64)
        _check(lib.crsd_dist_ranges(self._h, _p(r)))
        return r

    # ------------------------------------------------------------ introspection
    def info(self) -> dict:
        i = Info()
        _check(lib.crsd_get_info(self._h, ctypes.byref(i)))
        return {k: getattr(i, k) for k, _ in _INFO_FIELDS}

    def x_layout(self):
        lo, n, hi = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        _check(lib.crsd_dist_x_layout(self._h, ctypes.byref(lo), ctypes.byref(n), ctypes.byref(hi)))
        return lo.value, n.value, hi.value

    def jit_source(self) -> str:
        """CUDA source of the JIT variant's per-pattern codelets."""
        n = ctypes.c_int64()
        _check(lib.crsd_jit_source(self._h, None, 0, ctypes.byref(n)))
        buf = ctypes.create_string_buffer(n.value + 1)
        _check(lib.crsd_jit_source(self._h, buf, n.value + 1, ctypes.byref(n)))
        return buf.value.decode()

    def jit_cubin(self) -> bytes:
        """The sm_100a cubin of the JIT codelets (compiled by NVRTC on demand;
        no GPU needed) -- for cuobjdump / nvdisasm inspection."""
        n = ctypes.c_int64()
        _check(lib.crsd_jit_cubin(self._h, None, 0, ctypes.byref(n)))
        buf = ctypes.create_string_buffer(n.value)
        _check(lib.crsd_jit_cubin(self._h, buf, n.value, ctypes.byref(n)))
        return buf.raw[: n.value]

    def last_launch_count(self) -> int:
        c = ctypes.c_int32()
        _check(lib.crsd_last_launch_count(self._h, ctypes.byref(c)))
        return c.value

    def export(self) -> dict:
        """Host copies of the CRSD structure, as the layout dict oracle.decode reads."""
        inf = self.info()
        ni, npat, nseg, ns = inf["ninst"], inf["npat"], inf["nseg"], inf["nscatter"]
        a = dict(
            inst_first_seg=np.empty(ni, np.int64),
            inst_nseg=np.empty(ni, np.int64),
            inst_pattern=np.empty(ni, np.int32),
            pat_ptr=np.empty(npat + 1, np.int64),
            pat_offsets=np.empty(max(inf["noffsets"], 1), np.int64),
            vals=np.empty(inf["nslots"], self.dtype),
            scat_ptr=np.empty(nseg + 1, np.int64),
            scat_row=np.empty(max(ns, 1), np.int32),
            scat_col=np.empty(max(ns, 1), np.int64),
            scat_val=np.empty(max(ns, 1), self.dtype),
        )
        e = Export(**{k: v.ctypes.data for k, v in a.items()})
        _check(lib.crsd_export(self._h, ctypes.byref(e)))
        a["pat_offsets"] = a["pat_offsets"][: inf["noffsets"]]
        a["scat_row"], a["scat_col"], a["scat_val"] = a["scat_row"][:ns], a["scat_col"][:ns], a["scat_val"][:ns]
        po = a["pat_offsets"]
        pp = a["pat_ptr"]
        a["inst_offsets"] = [po[pp[p] : pp[p + 1]].tolist() for p in a["inst_pattern"]]
        a.update(nrows=inf["row_end"] - inf["row_begin"], ncols=inf["ncols"], mrows=inf["mrows"])
        return a


class Comm:
    """NCCL communicator owned by libcrsd, bootstrapped over torch.distributed."""

    def __init__(self, rank: int, world: int, device: int, pg=None):
        import torch
        import torch.distributed as dist

        uid = np.zeros(128, np.uint8)
        if rank == 0:
            _check(lib.crsd_comm_unique_id(_p(uid)))
        t = torch.from_numpy(uid.copy())
        if dist.get_backend(pg) == "nccl":
            t = t.cuda(device)
        dist.broadcast(t, src=0, group=pg)
        uid = t.cpu().numpy().copy()
        h = ctypes.c_void_p()
        _check(lib.crsd_comm_init_rank(_p(uid), rank, world, device, ctypes.byref(h)))
        self._h = h

    def allreduce_f64(self, dev_tensor, stream=None):
        """In-place sum over ranks of a CUDA float64 tensor (crsd_comm_allreduce_f64: ncclAllReduce)."""
        _check(lib.crsd_comm_allreduce_f64(self._h, ctypes.c_void_p(dev_tensor.data_ptr()), dev_tensor.numel(), _stream_ptr(stream)))
        return dev_tensor

    def error(self) -> int:
        return 0

    def close(self):
        if self._h is not None and self._h.value:
            lib.crsd_comm_destroy(self._h)
        self._h = None


class P2PComm:
    """Peer-memory communicator owned by libcrsd (crsd_comm_init_p2p /
    crsd_comm_p2p_open): the halo exchange and the CG's scalar allreduce run
    as the library's own kernels over CUDA-IPC-mapped regions. Only the
    64-byte IPC handles and the range table travel over torch.distributed
    (any backend: gloo works, so several processes may share one GPU)."""

    def __init__(self, rank: int, world: int, device: int, mailbox_bytes: int = 64 << 20, pg=None):
        import torch
        import torch.distributed as dist

        self.rank, self.world, self.device, self._pg = rank, world, device, pg
        self._h = None
        # every step is collective: if any rank fails (no memory, no IPC
        # between the visible devices, ...) every rank raises, none waits
        # forever in the next exchange
        handle = np.zeros(65, np.uint8)  # 64-byte IPC handle + ok flag
        h = ctypes.c_void_p()
        err = None
        try:
            _check(lib.crsd_comm_init_p2p(rank, world, device, int(mailbox_bytes), _p(handle), ctypes.byref(h)))
            self._h = h
            handle[64] = 1
        except CRSDError as e:
            err = e
        allh = self._allgather(torch.from_numpy(handle.copy()))
        if not allh[:, 64].all():
            self.close()
            raise err if err is not None else CRSDError(1, "peer-memory init failed on another rank")
        try:
            _check(lib.crsd_comm_p2p_open(self._h, _p(np.ascontiguousarray(allh[:, :64]))))
        except CRSDError as e:
            err = e
        ok = self._allgather(torch.tensor([0 if err else 1], dtype=torch.int64))
        if not ok.all():
            self.close()
            raise err if err is not None else CRSDError(1, "peer-memory open failed on another rank")

    def _allgather(self, t):
        import torch
        import torch.distributed as dist

        dev = torch.device("cuda", self.device) if dist.get_backend(self._pg) == "nccl" else torch.device("cpu")
        t = t.to(dev)
        out = [torch.empty_like(t) for _ in range(self.world)]
        dist.all_gather(out, t, group=self._pg)
        return torch.stack(out).cpu().numpy()

    def allgather_i64(self, row: np.ndarray) -> np.ndarray:
        import torch

        return np.ascontiguousarray(self._allgather(torch.from_numpy(np.asarray(row, np.int64).copy())), np.int64)

    def allreduce_f64(self, dev_tensor, stream=None):
        """In-place sum over ranks of a CUDA float64 tensor with <= 4 elements (crsd_comm_allreduce_f64)."""
        _check(lib.crsd_comm_allreduce_f64(self._h, ctypes.c_void_p(dev_tensor.data_ptr()), dev_tensor.numel(), _stream_ptr(stream)))
        return dev_tensor

    def error(self) -> int:
        """0, or 1/2/3 when a send / recv / allreduce wait timed out (crsd_comm_error)."""
        e = ctypes.c_int32()
        _check(lib.crsd_comm_error(self._h, ctypes.byref(e)))
        return e.value

    def close(self):
        if self._h is not None and self._h.value:
            lib.crsd_comm_destroy(self._h)
        self._h = None


def dist_plan(world: int, rank: int, ranges4: np.ndarray):
    """Host-only halo plan (crsd_dist_plan): returns (recv, send) lists of (peer, begin, count)."""
    r = np.ascontiguousarray(ranges4, dtype=np.int64).reshape(world, 4)
    cap = 2 * world
    bufs = [np.zeros(cap, np.int64) for _ in range(6)]
    nr, ns = ctypes.c_int64(), ctypes.c_int64()
    _check(lib.crsd_dist_plan(world, rank, _p(r), _p(bufs[0]), _p(bufs[1]), _p(bufs[2]), ctypes.byref(nr), _p(bufs[3]), _p(bufs[4]), _p(bufs[5]), ctypes.byref(ns)))
    recv = list(zip(bufs[0][: nr.value].tolist(), bufs[1][: nr.value].tolist(), bufs[2][: nr.value].tolist()))
    send = list(zip(bufs[3][: ns.value].tolist(), bufs[4][: ns.value].tolist(), bufs[5][: ns.value].tolist()))
    return recv, send


def partition_rows(nrows: int, mrows: int, world: int, weights: Optional[np.ndarray] = None) -> np.ndarray:
    b = np.zeros(world + 1, np.int64)
    w = None if weights is None else np.ascontiguousarray(weights, dtype=np.float64)
    _check(lib.crsd_partition_rows(nrows, mrows, world, _p(w) if w is not None else None, _p(b)))
    return b


def version() -> str:
    return lib.crsd_version().decode()
