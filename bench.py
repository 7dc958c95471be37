#!/usr/bin/env python
"""Benchmark of the CRSD SpMV hot path on B200 (driver contract: one JSON line).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c1..c5]
                    [--dtype f64|f32] [--impl crsd|reference] [--workload spmv|cg]

Metric (BASELINE.json): CRSD SpMV GFLOP/s (2 nnz / t, whole job) with the
achieved HBM GB/s on algorithmic bytes and its fraction of the measured B200
copy bandwidth (MEASURED_PEAKS.json), at 1/2/4/8 GPUs.

A step is one y = A x (alpha 1, beta 0: the paper's SpMV) over
the whole workload, inputs resident in HBM. Default workload at EVERY N:
BASELINE.json config 5, the 3D 7-point Laplacian on 768^3 (452,984,832 rows,
3.17e9 nonzeros, fp64) -- strong scaling: N ranks own N row blocks of the one
matrix, x halos move between ranks inside crsd_spmv_dist (the library's
peer-memory kernels over NVLink, NCCL send/recv fallback), overlapped with
the interior segments. At N = 1 the same run also times the north-star
matrix, config 3 (27-point 192^3 with idle sections and 0.1 % scatter
points) in fp64 and fp32, each with its own roofline record.

When N > 1 and WORLD_SIZE is unset the script re-launches itself under
torch.distributed.run with N ranks (one per GPU, rendezvous on 127.0.0.1).

--impl reference times the oracle (oracle/coo_native.c: the definition
accumulated in the matrix dtype, OpenMP over row ranges of the row-sorted
COO, all host cores) on a bounded row sample of the same workload: the tier's
reference arm. Under torchrun only rank 0 runs it.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "CRSD SpMV GFLOP/s and achieved HBM GB/s (% of B200 peak) at 1/2/4/8 GPUs"
L2_BYTES = 126 * 1024 * 1024
VARIANTS = {"auto": 0, "ldg": 1, "tma": 2, "pipe": 3, "jit": 4}
VNAME = {1: "ldg", 2: "tma", 3: "pipe", 4: "jit"}
KNAME = {1: "crsd_spmv_ldg", 2: "crsd_spmv_tma", 3: "crsd_spmv_pipe", 4: "crsd_jit"}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            j = json.load(f)
        return float(j.get("hbm_gbs", 6650.0)), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def _affinity():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


# read once at import: OMP_PROC_BIND later pins the main thread to one core
_HOST_CORES = _affinity()


def host_cores():
    return _HOST_CORES


def host_cpu_info():
    info = {"nproc": host_cores()}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            k, _, v = line.partition(":")
            k, v = k.strip(), v.strip()
            if k == "Model name":
                info["model"] = v
            elif k == "Socket(s)":
                info["sockets"] = int(v) if v.isdigit() else v
            elif k == "Thread(s) per core":
                info["threads_per_core"] = int(v) if v.isdigit() else v
    except Exception:
        pass
    return info


# ---------------------------------------------------------------- workloads
def _stencil_disps(kind, dims):
    from gen import matrices

    disps = matrices._disps(kind)
    lin = [di + dims[0] * (dj + dims[1] * dk) for (di, dj, dk) in disps]
    return [disps[q] for q in np.argsort(lin, kind="stable")]


def rank_rows(cfg, world, rank, mrows=256):
    """Global size and this rank's row block [rb, re)."""
    from paper_conf_icpp_sunzwzyr11_b200 import partition_rows

    if cfg == "c5":
        N = 768**3
        b = partition_rows(N, mrows, world)  # uniform rows: equal blocks are byte-balanced
    elif cfg == "c2":
        N = 256**3 * world  # weak: a 256^3 slab per rank
        b = [k * 256**3 for k in range(world + 1)]
    elif cfg == "c4":
        import gen

        N = 100_000_000
        if world == 1:
            b = [0, N]
        else:
            # byte-balanced row blocks (equal rows give
            # max/avg 1.52 on C4): weight per row = its stored diagonals + x + y
            w = np.empty(N, np.float64)
            for r0, r1, offs in gen.matrices.c4_ranges(N):
                w[r0:r1] = len(offs) + 2
            b = partition_rows(N, 512, world, w)
            del w
    else:
        raise SystemExit(f"config {cfg} is one-GPU only")
    return N, int(b[rank]), int(b[rank + 1])


def coo_matrix(cfg, dtype):
    """The whole single-GPU workload `cfg` as a COO (gen.COO; values in the
    dtype) -- for scripts that build several handles of one matrix."""
    import gen

    dt = np.float64 if dtype == "f64" else np.float32
    a = {
        "c1": gen.config1,
        "c2": gen.config2,
        "c3": gen.config3,
        "c3ns": lambda: gen.config3(scatter_frac=0.0),
        "c4": gen.config4,
        "c5": gen.config5,
    }[cfg]()
    return gen.COO(a.nrows, a.ncols, a.row, a.col, a.val.astype(dt))


def build(cfg, dtype, world, rank, dev, mrows=0, variant=0, nthreads=0):
    """Build this rank's CRSD handle for config `cfg`. Large configs are
    generated as CSR by gen/fastgen.c and handed to crsd_create_from_csr,
    which reads canonical CSR in place (C5 holds 3.17e9 entries).
    Returns (A, description, (rb, re), N global rows, build seconds)."""
    import gen
    from gen import fast
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix

    dt = np.float64 if dtype == "f64" else np.float32
    kw = dict(device=dev, mrows=mrows, variant=variant, nthreads=nthreads)
    t0 = time.perf_counter()
    if cfg in ("c1", "c3", "c3ns"):
        if world != 1:
            raise SystemExit(f"config {cfg} is a single-GPU workload")
        if cfg == "c1":
            a = gen.config1()
            desc = f"C1: 2D 5-point Laplacian 64x64 (4,096 rows) + 16 scatter points, {dtype} (L2-resident: latency, L2 flushed before every step)"
        else:
            # c3ns: the same matrix without its scatter points (diagnostic only)
            a = gen.config3(scatter_frac=0.001 if cfg == "c3" else 0.0)
            desc = f"C3: 3D 27-point FVM stencil 192^3 with idle sub-blocks and {'0.1% scatter points' if cfg == 'c3' else 'no scatter points'} ({a.nrows:,} rows), {dtype}"
        A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val.astype(dt), **kw)
        N, rb, re = a.nrows, 0, a.nrows
        del a
    else:
        N, rb, re = rank_rows(cfg, world, rank)
        if cfg == "c4":
            ptr, col, val = fast.band(N, gen.matrices.c4_ranges(N), 4, rb, re, nthreads=nthreads, csr=True)
            desc = f"C4: banded, 19 offsets in 9 groups / 4 patterns, 100M rows, {dtype}"
        elif cfg == "c5":
            if dtype != "f64":
                raise SystemExit("config c5 is fp64")
            d = (768, 768, 768)
            ptr, col, val = fast.stencil(d, _stencil_disps("7pt", d), False, False, 5, None, rb, re, nthreads=nthreads, csr=True)
            desc = f"C5: 3D 7-point Laplacian 768^3 ({N:,} rows, 3,167,354,880 nonzeros), fp64"
        else:  # c2
            d = (256, 256, 256 * world)
            ptr, col, val = fast.stencil(d, _stencil_disps("7pt", d), False, True, 2, None, rb, re, nthreads=nthreads, csr=True)
            desc = f"C2: 3D 7-point FDM Laplacian 256^3 per GPU (grid 256x256x{256 * world}, {N:,} rows), {dtype}"
        if dt != np.float64:
            val = val.astype(dt)
        A = CRSDMatrix.from_csr(N, N, ptr, col, val, row_range=None if (rb, re) == (0, N) else (rb, re), **kw)
        del ptr, col, val
    return A, desc, (rb, re), N, time.perf_counter() - t0


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""

    FIELDS = "clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap"

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE,
                stderr=subprocess.DEVNULL,
                text=True,
            )
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            time.sleep(0.3)
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) == 7:
                self.samples.append(parts)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for s in self.samples:
            for nm, v in zip(names, s[3:]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.samples)}


def copy_bandwidth(dev, reps=5):
    """Same recipe as MEASURED_PEAKS.json: torch copy of 1 Gi bf16 elements,
    read+write bytes, best of `reps` (context for this box's HBM)."""
    import torch

    a = torch.empty(1 << 30, dtype=torch.bfloat16, device=f"cuda:{dev}")
    b = torch.empty_like(a)
    best = 0.0
    for _ in range(reps + 1):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        b.copy_(a)
        e.record()
        e.synchronize()
        best = max(best, 2 * a.numel() * 2 / (s.elapsed_time(e) * 1e-3) / 1e9)
    del a, b
    torch.cuda.empty_cache()
    return round(best, 1)


def read_bandwidth(nbytes=16 << 30, reps=5):
    """Read-only HBM bandwidth on this box (tools/hbm_read.cu: a grid-stride
    stream of 128-bit loads, best of `reps` passes over 16 GiB) -- context for
    a read-dominated kernel whose fraction of the read + write copy peak can
    exceed 1. None when the probe is not built."""
    import ctypes

    lib = os.path.join(ROOT, "tools", "libhbmread.so")
    if not os.path.exists(lib):
        return None
    f = ctypes.CDLL(lib).hbm_read_gbs
    f.argtypes, f.restype = [ctypes.c_int64, ctypes.c_int], ctypes.c_double
    g = f(nbytes, reps)
    return round(g, 1) if g > 0 else None


def load_traffic(key):
    """ncu dram bytes (read + write) per launch of the dominant kernel on this
    workload, from one `ncu --set full` capture (profiles/traffic.json, keyed
    "<config>_<dtype>_<kernel>"); None when that kernel was not captured."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f).get(key)
    return None


# ---------------------------------------------------------------- timing
def timed_steps(step, steps, stream, count):
    """K steps back to back between two CUDA events on the launching stream
    (no per-step host work besides the launches themselves). Returns (ms per
    step, whole-region ms, kernel launches)."""
    import torch

    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0.record(stream)
    for _ in range(steps):
        step()
    t1.record(stream)
    launches = steps * count()  # every step launches the same kernels
    torch.cuda.synchronize()
    total = t0.elapsed_time(t1)
    return total / steps, total, launches


def sub_record(cfg, dtype, args, dev):
    """One-GPU timing of another BASELINE matrix inside the same run (the
    north-star C3 records at N = 1): value, ms, roofline of its own."""
    import torch

    A, desc, _, N, bs = build(cfg, dtype, 1, 0, dev, mrows=0, variant=VARIANTS[args.variant])
    info = A.info()
    tdt = torch.float64 if dtype == "f64" else torch.float32
    x = torch.from_numpy(np.random.default_rng(7).uniform(-1, 1, N)).to(f"cuda:{dev}", tdt)
    y = torch.empty(N, dtype=tdt, device=f"cuda:{dev}")
    stream = torch.cuda.current_stream()

    def step():
        A.spmv(x, y, 1.0, 0.0)

    # a sub-record's steps are short (0.1-0.8 ms): at least 200 of them, so
    # the timed region is not dominated by its ramp-up
    steps = max(args.steps, 200)
    for _ in range(max(args.warmup, 10)):
        step()
    torch.cuda.synchronize()
    clk = ClockSampler(dev).start()
    ms, total_ms, launches = timed_steps(step, steps, stream, A.last_launch_count)
    clocks = clk.stop()
    ub = info["unique_bytes_beta0"]
    peak, _ = measured_peaks()
    achieved = ub / (ms * 1e-3) / 1e9
    kname = KNAME[info["variant"]] + ("_rs" if info.get("regstage") else "")
    rec = {
        "workload": desc,
        "value": round(2.0 * info["nnz"] / (ms * 1e-3) / 1e9, 3),
        "unit": "GFLOP/s",
        "ms_per_step": round(ms, 5),
        "dtype": dtype,
        "nnz": info["nnz"],
        "mrows": info["mrows"],
        "kernel_variant": VNAME[info["variant"]],
        "scatter": info["nscatter"],
        "fills": info["nfills"],
        "steps": steps,
        "launches_per_step": round(launches / steps, 2),
        "roofline": {
            "bound": "hbm", "kernel": kname, "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 4), "traffic": load_traffic(f"{cfg}_{dtype}_{kname}"),
            "algorithmic_bytes_per_launch": int(ub), "avg_step_ms": round(ms, 5),
        },
        "l2": f"inputs larger than L2 ({ub / 1e9:.2f} GB per step); no flush",
        "build_s": round(bs, 1),
        "clocks": clocks,
    }
    A.close()
    del x, y
    torch.cuda.empty_cache()
    if not args.no_cpu:
        # the oracle's native loop on the WHOLE matrix for C1-C3 (BASELINE.md
        # §4), a 200 M-entry row prefix for the larger ones
        rec["cpu_baseline"] = cpu_baseline(cfg, dtype, cap_nnz=(1 << 62) if cfg in ("c1", "c2", "c3") else 200_000_000)
    return rec


# ---------------------------------------------------------------- CPU baseline
def cpu_sample(cfg, dtype, cap_nnz):
    """Rows [0, cut) of the workload with about cap_nnz entries, as a
    row-sorted COO (the reference arm and cpu_baseline generate only these).
    Returns (nrows, ncols, cut, row, col, val, nnz of the whole matrix)."""
    import gen
    from gen import fast

    dt = np.float64 if dtype == "f64" else np.float32
    if cfg in ("c1", "c3", "c3ns"):
        a = gen.config1() if cfg == "c1" else gen.config3(scatter_frac=0.001 if cfg == "c3" else 0.0)
        a = a.sorted()
        N = a.nrows
        cut = N if a.nnz <= cap_nnz else max(1, int(N * cap_nnz // a.nnz))
        m = a.row < cut
        return N, N, cut, a.row[m], a.col[m], a.val[m].astype(dt), a.nnz
    N, _, _ = rank_rows(cfg, 1, 0)
    per_row = {"c5": 7.0, "c2": 7.0, "c4": 11.9}[cfg]
    cut = int(min(N, max(1024, cap_nnz / per_row)))
    if cfg == "c4":
        r, c, v = fast.band(N, gen.matrices.c4_ranges(N), 4, 0, cut)
        total = 1_186_000_000
    else:
        d = (768, 768, 768) if cfg == "c5" else (256, 256, 256)
        r, c, v = fast.stencil(d, _stencil_disps("7pt", d), False, cfg == "c2", 5 if cfg == "c5" else 2, None, 0, cut)
        total = 3_167_354_880 if cfg == "c5" else 117_047_296
    return N, N, cut, r, c, v.astype(dt), total


def time_native(nrows, r, c, v, x, nthreads, reps=5):
    """Median of `reps` runs of the oracle's native-dtype loop (after one warm-up)."""
    from oracle import coo as oracle_coo

    y = np.empty(nrows, dtype=v.dtype)
    oracle_coo.coo_spmv_native(nrows, r, c, v, x, nthreads=nthreads, out=y)
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter()
        oracle_coo.coo_spmv_native(nrows, r, c, v, x, nthreads=nthreads, out=y)
        ts.append(time.perf_counter() - t0)
    return statistics.median(ts)


def cpu_baseline(cfg, dtype, cap_nnz=200_000_000):
    """The oracle's plain COO SpMV in the matrix dtype (oracle/coo_native.c,
    as it stands) on the host cores, on a bounded row sample of the workload:
    1 thread and all cores (OpenMP over row ranges, OMP_PROC_BIND=spread),
    median of 5 each."""
    N, ncols, cut, r, c, v, total = cpu_sample(cfg, dtype, cap_nnz)
    x = np.random.default_rng(7).uniform(-1, 1, ncols).astype(v.dtype)
    k = r.shape[0]
    cores = host_cores()
    t1 = time_native(cut, r, c, v, x, 1)
    tn = time_native(cut, r, c, v, x, cores)
    return {
        "value": round(2.0 * k / tn / 1e9, 3),
        "unit": "GFLOP/s",
        "cores": cores,
        "kind": "oracle",
        "sample": f"rows [0,{cut:,}) of the workload ({k:,} nonzeros, {k / total:.1%} of the matrix); oracle/coo_native.c "
                  f"(definition in the matrix dtype, OpenMP over row ranges of the row-sorted COO, OMP_PROC_BIND=spread), median of 5",
        "value_1_thread": round(2.0 * k / t1 / 1e9, 3),
        "host": host_cpu_info(),
    }


# ---------------------------------------------------------------- reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return  # the oracle arm runs on rank 0 alone; the other ranks exit without work
    from oracle import coo as oracle_coo

    cores = host_cores()
    # bounded sample: calibrate the oracle's rate on a small sample, then size
    # each step so the whole --steps/--warmup run stays within ~2 minutes
    budget = float(os.environ.get("CRSD_REF_BUDGET_S", "120"))
    N, ncols, cut, r, c, v, total = cpu_sample(args.config, args.dtype, 20_000_000)
    x = np.random.default_rng(7).uniform(-1, 1, ncols).astype(v.dtype)
    t = time_native(cut, r, c, v, x, cores, reps=2)
    rate = r.shape[0] / max(t, 1e-6)
    cap = int(min(total, 500_000_000, max(10_000_000, rate * budget / (args.steps + args.warmup))))
    if cap > r.shape[0]:
        del r, c, v
        N, ncols, cut, r, c, v, total = cpu_sample(args.config, args.dtype, cap)
        x = np.random.default_rng(7).uniform(-1, 1, ncols).astype(v.dtype)
    k = r.shape[0]
    y = np.empty(cut, dtype=v.dtype)
    for _ in range(args.warmup):
        oracle_coo.coo_spmv_native(cut, r, c, v, x, nthreads=cores, out=y)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle_coo.coo_spmv_native(cut, r, c, v, x, nthreads=cores, out=y)
        ts.append(time.perf_counter() - t0)
    tm = statistics.mean(ts)
    gflops = 2.0 * k / tm / 1e9
    sample = (f"rows [0,{cut:,}) of the workload, {k:,} nonzeros per step ({k / total:.1%} of the matrix); "
              f"oracle/coo_native.c on {cores} host threads")
    line = {
        "impl": "reference",
        "metric": METRIC,
        "value": round(gflops, 4),
        "unit": "GFLOP/s",
        "n_gpus": args.gpus,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(tm * 1e3, 3),
        "higher_is_better": True,
        "scaling": "strong" if args.config in ("c4", "c5") else "weak",
        "vs_baseline": None,
        "dtype": args.dtype,
        "data": "synthetic",
        "config": {"workload": args.config.upper() + " (row sample, see cpu_baseline.sample)", "alpha": 1.0, "beta": 0.0},
        "cpu_baseline": {"value": round(gflops, 4), "unit": "GFLOP/s", "cores": cores, "kind": "oracle", "sample": sample,
                         "host": host_cpu_info()},
        "e2e": {"value": round(gflops, 4), "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- CRSD arm
def init_dist(args):
    import torch
    import torch.distributed as dist

    world = args.gpus
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    local_world = int(os.environ.get("LOCAL_WORLD_SIZE", str(world)))
    # --share-gpu: every rank on cuda:0 (functional check of the multi-rank
    # path on a one-GPU box; NCCL refuses two ranks per GPU, so the torch
    # plumbing uses gloo and the transport must be p2p). Not a scaling number.
    if args.share_gpu:
        local_rank = 0
        if args.transport == "nccl":
            raise SystemExit("--share-gpu needs the p2p transport")
    if world > 1:
        dist.init_process_group("gloo" if args.share_gpu else "nccl", init_method="env://")
        world, rank = dist.get_world_size(), dist.get_rank()
    torch.cuda.set_device(local_rank)
    nthreads = max(1, host_cores() // max(1, local_world))
    return world, rank, local_rank, nthreads


def make_comm(args, A, rank, world, dev, es):
    from paper_conf_icpp_sunzwzyr11_b200 import Comm, P2PComm

    lo, _, hi = A.x_layout()
    comm, transport = None, None
    if args.transport in ("auto", "p2p"):
        try:
            comm, transport = P2PComm(rank, world, dev, mailbox_bytes=max(1 << 20, 4 * (lo + hi) * es)), "p2p"
        except Exception as e:  # collective: every rank lands here together
            if args.transport == "p2p":
                raise
            print(f"[bench] peer-memory transport unavailable ({e}); using NCCL", file=sys.stderr)
    if comm is None:
        comm, transport = Comm(rank, world, dev), "nccl"
    A.dist_bind(comm)
    return comm, transport


def run_spmv(args):
    import torch
    import torch.distributed as dist

    world, rank, dev, nthreads = init_dist(args)
    red_dev = "cpu" if args.share_gpu else f"cuda:{dev}"
    A, desc, (rb, re), N, build_s = build(args.config, args.dtype, world, rank, dev, args.mrows, VARIANTS[args.variant], nthreads)
    info = A.info()
    dt = np.float64 if args.dtype == "f64" else np.float32
    tdt = torch.float64 if args.dtype == "f64" else torch.float32
    es = np.dtype(dt).itemsize
    stream = torch.cuda.current_stream()
    nloc = re - rb
    x_own = torch.from_numpy(np.random.default_rng(7 + rank).uniform(-1, 1, nloc).astype(dt)).to(f"cuda:{dev}")
    comm, transport = None, None
    if world > 1:
        comm, transport = make_comm(args, A, rank, world, dev, es)
        lo, _, hi = A.x_layout()
        if transport == "p2p":
            # the library-owned padded x, mapped by the neighbours: halos
            # arrive as one-sided puts, received inside the boundary kernel
            xp = A.dist_x_alloc(comm)
            transport = "p2p one-sided puts"
        else:
            xp = torch.zeros(lo + nloc + hi, dtype=tdt, device=f"cuda:{dev}")
        xp[lo : lo + nloc] = x_own
        y = torch.empty(nloc, dtype=tdt, device=f"cuda:{dev}")

        def step():
            A.spmv_dist(xp, y, 1.0, 0.0, comm)
    else:
        y = torch.empty(N, dtype=tdt, device=f"cuda:{dev}")

        def step():
            A.spmv(x_own, y, 1.0, 0.0)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if comm is not None and comm.error():
        raise SystemExit(f"[bench] rank {rank}: a peer-memory wait timed out during warm-up (code {comm.error()}); no valid number")

    # timed region: K steps, per-step CUDA events on the launching stream,
    # barrier + synchronize on both sides
    # C1 fits in L2 (0.23 MB): flush it (write a buffer > L2) before every
    # step, outside the step's events; the metric is then the per-step time
    flush = torch.empty(2 * L2_BYTES // 4, dtype=torch.int32, device=f"cuda:{dev}") if args.config == "c1" else None
    clk = ClockSampler(dev).start()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    if flush is None:
        step_ms, total_ms, launches = timed_steps(step, args.steps, stream, A.last_launch_count)
        step_ms = [step_ms]
    else:  # per-step events, the flush outside them
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        for i in range(args.steps):
            flush.zero_()
            ev[i][0].record(stream)
            step()
            ev[i][1].record(stream)
        torch.cuda.synchronize()
        step_ms = [s_.elapsed_time(e_) for s_, e_ in ev]
        total_ms, launches = sum(step_ms), args.steps * A.last_launch_count()
    if world > 1:
        dist.barrier()
    clocks = clk.stop()
    if comm is not None and comm.error():
        raise SystemExit(f"[bench] rank {rank}: a peer-memory wait timed out in the timed region (code {comm.error()}); no valid number")
    nnz_local, ub = info["nnz"], info["unique_bytes_beta0"]
    if world > 1:
        tt = torch.tensor([total_ms, statistics.mean(step_ms)], dtype=torch.float64, device=red_dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        total_ms, kern_ms = float(tt[0].item()), float(tt[1].item())
        nn = torch.tensor([nnz_local, ub, launches], dtype=torch.float64, device=red_dev)
        dist.all_reduce(nn)
        nnz_all, ub_all, launches_all = (float(v) for v in nn.tolist())
    else:
        kern_ms = statistics.mean(step_ms)
        nnz_all, ub_all, launches_all = float(nnz_local), float(ub), float(launches)
    ms = total_ms / args.steps
    if flush is not None:
        ms = kern_ms = statistics.median(step_ms)
    gflops = 2.0 * nnz_all / (ms * 1e-3) / 1e9
    peak, peak_src = measured_peaks()
    achieved = ub_all / world / (kern_ms * 1e-3) / 1e9  # per GPU: whole-job bytes / N / max-over-ranks step time

    # e2e through the public C-ABI with host buffers (pinned)
    e2e = run_e2e(args, A, world, rank, dev, dt, tdt, N, rb, re, nnz_all, red_dev, comm, transport,
                  xp if world > 1 else None)
    if rank != 0:
        if comm is not None:
            comm.close()
        dist.destroy_process_group()
        return

    subs = None
    other = None
    cpu = None
    if world == 1 and args.config == "c5" and not args.no_sub:
        # the north-star matrix (BASELINE config 3) in both precisions
        A.close()
        del x_own, y
        torch.cuda.empty_cache()
        subs = {"f64": sub_record("c3", "f64", args, dev), "f32": sub_record("c3", "f32", args, dev)}
        # BASELINE config 4 on one GPU (the 2/4/8-GPU strong-scaling band)
        other = {"c4_f32": sub_record("c4", "f32", args, dev)}
    if world == 1 and not args.no_cpu:
        cpu = cpu_baseline(args.config, args.dtype)
    box_copy = copy_bandwidth(dev)
    box_read = read_bandwidth()
    kname = KNAME[info["variant"]] + ("_rs" if info.get("regstage") else "")
    line = {
        "metric": METRIC,
        "value": round(gflops, 3),
        "unit": "GFLOP/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(ms, 5),
        "higher_is_better": True,
        "scaling": "strong" if args.config in ("c4", "c5") else "weak",
        "vs_baseline": None,
        "dtype": args.dtype,
        "data": "synthetic",
        "config": {
            "workload": desc,
            "nnz": int(nnz_all),
            "rows_per_rank": int(re - rb),
            "mrows": info["mrows"],
            "kernel_variant": VNAME[info["variant"]],
            "alpha": 1.0,
            "beta": 0.0,
            "patterns": info["npat"],
            "instances": info["ninst"],
            "fills": info["nfills"],
            "scatter": info["nscatter"],
            "l2": (f"inputs larger than L2 ({ub_all / 1e9:.2f} GB streamed per step vs {L2_BYTES / 2**20:.0f} MiB L2); no flush" if flush is None else f"L2 flushed (252 MiB written) before every step; ms_per_step = median per-step CUDA-event time"),
            "build_s": round(build_s, 1),
            "parallelism": f"row-partitioned x{world}" + (f", {transport} halo" if world > 1 else "") + (", ranks share cuda:0 (functional only)" if args.share_gpu else ""),
        },
        "latency_us": round(ms * 1e3, 2) if flush is not None else None,
        "hbm_gbs": round(ub_all / (ms * 1e-3) / 1e9, 1),
        "hbm_frac_of_peak": round(ub_all / (ms * 1e-3) / 1e9 / (peak * world), 4),
        "roofline": {
            "bound": "hbm",
            "kernel": kname,
            "achieved": round(achieved, 1),
            "peak": peak,
            "peak_source": peak_src,
            "unit": "GB/s",
            "frac": round(achieved / peak, 4),
            "traffic": load_traffic(f"{args.config}_{args.dtype}_{kname}") if (world == 1 and not args.mrows) else None,
            "algorithmic_bytes_per_launch": int(ub_all / world),
            "avg_launch_ms": round(kern_ms, 5),
            "launches_per_step": round(launches_all / world / max(1, args.steps), 2),
            "scope": "per GPU: whole-job algorithmic bytes / N / the max-over-ranks CUDA-event step time; with several launches per step (occupancy-class ranges, interior/boundary) the step's bytes / the step's time",
            "copy_gbs_this_box": box_copy,
            "read_gbs_this_box": box_read,
            "frac_of_this_box_read": round(achieved / box_read, 4) if box_read else None,
        },
        "north_star_c3": subs,
        "other_configs": other,
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": int(launches_all),
        "clocks": clocks,
    }
    print(json.dumps(line), flush=True)
    if comm is not None:
        comm.close()
    if world > 1:
        dist.destroy_process_group()


def run_e2e(args, A, world, rank, dev, dt, tdt, N, rb, re, nnz_all, red_dev, comm, transport, xp=None):
    """The metric end to end through the public C-ABI: every step copies the
    step's x from pinned host memory and its y back (N = 1: crsd_spmv_host,
    the library's chunked H2D / SpMV / D2H pipeline; N > 1: per rank the
    owned x slice in, crsd_spmv_dist, the y slice out, max over ranks)."""
    import torch
    import torch.distributed as dist

    es = np.dtype(dt).itemsize
    ke = max(3, min(args.steps, 10))
    if world == 1:
        xh = torch.from_numpy(np.random.default_rng(7).uniform(-1, 1, N).astype(dt)).pin_memory()
        yh = torch.empty(N, dtype=tdt).pin_memory()
        for _ in range(2):
            A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr(), 1.0, 0.0)
        t0 = time.perf_counter()
        for _ in range(ke):
            A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr(), 1.0, 0.0)
        te = (time.perf_counter() - t0) / ke
        # the copy bound of the e2e step: H2D and D2H at the same time on two streams
        xd = torch.empty(N, dtype=tdt, device=f"cuda:{dev}")
        yd = torch.empty(N, dtype=tdt, device=f"cuda:{dev}")
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(3):
            with torch.cuda.stream(s1):
                xd.copy_(xh, non_blocking=True)
            with torch.cuda.stream(s2):
                yh.copy_(yd, non_blocking=True)
        torch.cuda.synchronize()
        bidir_ms = (time.perf_counter() - t0) / 3 * 1e3
        del xd, yd, xh, yh
        torch.cuda.empty_cache()
        return {
            "value": round(2.0 * nnz_all / te / 1e9, 3),
            "unit": "GFLOP/s",
            "h2d_bytes_per_step": int(N * es),
            "d2h_bytes_per_step": int(N * es),
            "ms_per_step": round(te * 1e3, 3),
            "concurrent_h2d_d2h_ms": round(bidir_ms, 3),
            "frac_of_copy_bound": round(bidir_ms / (te * 1e3), 3),
            "path": "crsd_spmv_host: chunked H2D(x) / SpMV / D2H(y) pipeline on three streams",
        }
    nloc = re - rb
    lo, _, hi = A.x_layout()
    y = torch.empty(nloc, dtype=tdt, device=f"cuda:{dev}")
    xh = torch.from_numpy(np.random.default_rng(7 + rank).uniform(-1, 1, nloc).astype(dt)).pin_memory()
    yh = torch.empty(nloc, dtype=tdt).pin_memory()

    def e2e_step():
        xp[lo : lo + nloc].copy_(xh, non_blocking=True)
        A.spmv_dist(xp, y, 1.0, 0.0, comm)
        yh.copy_(y, non_blocking=True)
        torch.cuda.current_stream().synchronize()

    for _ in range(2):
        e2e_step()
    dist.barrier()
    t0 = time.perf_counter()
    for _ in range(ke):
        e2e_step()
    te = torch.tensor([(time.perf_counter() - t0) / ke], dtype=torch.float64, device=red_dev)
    dist.all_reduce(te, op=dist.ReduceOp.MAX)
    te = float(te.item())
    return {
        "value": round(2.0 * nnz_all / te / 1e9, 3),
        "unit": "GFLOP/s",
        "h2d_bytes_per_step": int(N * es),
        "d2h_bytes_per_step": int(N * es),
        "ms_per_step": round(te * 1e3, 3),
        "path": f"per rank: H2D of the owned x slice, crsd_spmv_dist ({transport} halo + SpMV), D2H of the y slice; max over ranks",
    }


# ---------------------------------------------------------------- CG workload
def run_cg(args):
    """--workload cg: K steps of crsd_cg (textbook CG on the CRSD SpMV,
    SURVEY.md §8(f) NEXT 2) on the 7-point Dirichlet Laplacian of C2's grid
    (256^3 per GPU, SPD, exact values). A step = SpMV + 3 vector kernels; its
    algorithmic bytes are the SpMV's unique bytes + the vector traffic
    (DESIGN.md §13). N > 1: weak scaling, grid 256 x 256 x 256N cut into
    z-slabs, halo exchange + allreduced dots through the communicator
    (peer-memory kernels: graph batches; NCCL fallback: direct calls)."""
    import torch
    import torch.distributed as dist

    import gen
    from oracle import cg_ref
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix

    world, rank, local_rank, nthreads = init_dist(args)
    dev = f"cuda:{local_rank}"
    red_dev = "cpu" if args.share_gpu else dev
    dt = np.float64 if args.dtype == "f64" else np.float32
    tdt = torch.float64 if dt == np.float64 else torch.float32
    es = np.dtype(dt).itemsize
    n = 256
    nloc = n * n * n
    rb, re = rank * nloc, (rank + 1) * nloc
    N = nloc * world
    if world == 1:
        a = gen.spd_stencil_scatter((n, n, n), "7pt").astype(dt)
    else:
        a = gen.stencil((n, n, n * world), "7pt", row_begin=rb, row_end=re)
        a = gen.COO(N, N, a.row, a.col, a.val.astype(dt))
    kw = {"mrows": args.mrows} if args.mrows else {}
    if world > 1:
        kw["row_range"] = (rb, re)
    A = CRSDMatrix.from_coo(N, N, a.row, a.col, a.val, device=local_rank, tune=args.tune, **kw)
    info = A.info()
    comm, transport = None, None
    if world > 1:
        comm, transport = make_comm(args, A, rank, world, local_rank, es)
    step_bytes = info["unique_bytes_beta0"] + 10 * nloc * es
    nnz_local = int(a.nnz)
    step_flops = 2.0 * nnz_local + 10.0 * nloc
    rng = np.random.default_rng(17 + rank)
    bh = torch.from_numpy(rng.uniform(-1, 1, nloc).astype(dt)).pin_memory()
    b = bh.to(dev)
    x = torch.zeros(nloc, dtype=tdt, device=dev)
    K = args.steps
    check = min(K, 50)
    clocks = ClockSampler(local_rank).start()
    # warm-up: >= 300 steps (a short CG run otherwise starts below full clocks)
    A.cg(b, x, max(args.warmup, 300), 0.0, check_every=check, comm=comm)
    torch.cuda.synchronize()
    x.zero_()
    s_ev, e_ev = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    s_ev.record()
    res = A.cg(b, x, K, 0.0, check_every=check, comm=comm)
    e_ev.record()
    e_ev.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    ms = s_ev.elapsed_time(e_ev) / res["iterations"]
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=red_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    peak, peak_src = measured_peaks()
    achieved = step_bytes / (ms * 1e-3) / 1e9
    # e2e: pinned b -> device, K steps, x -> pinned host, every solve
    xh = torch.empty(nloc, dtype=tdt).pin_memory()
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    bd = bh.to(dev, non_blocking=True)
    xd = torch.zeros(nloc, dtype=tdt, device=dev)
    r2 = A.cg(bd, xd, K, 0.0, check_every=check, comm=comm)
    xh.copy_(xd, non_blocking=True)
    torch.cuda.synchronize()
    te = time.perf_counter() - t0
    if world > 1:
        t = torch.tensor([te], dtype=torch.float64, device=red_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        te = float(t.item())
        if comm is not None and comm.error():
            raise SystemExit("peer-memory wait timed out")
    if rank != 0:
        comm.close()
        dist.destroy_process_group()
        return
    cpu = None
    if world == 1 and not args.no_cpu:
        # cpu_baseline: the CG oracle as it stands on a bounded sample (64^3 grid)
        ns = 64
        a_s = gen.spd_stencil_scatter((ns, ns, ns), "7pt").astype(dt)
        b_s = rng.uniform(-1, 1, a_s.nrows)
        ks = 5
        t0 = time.perf_counter()
        cg_ref.cg(a_s, b_s, np.zeros(a_s.nrows), ks)
        tc = (time.perf_counter() - t0) / ks
        cpu = {
            "value": round((2.0 * a_s.nnz + 10.0 * a_s.nrows) / tc / 1e9, 4),
            "unit": "GFLOP/s",
            "cores": 1,
            "kind": "oracle",
            "sample": f"oracle/cg_ref.py (long-double definition SpMV + numpy dots), 7-pt 64^3 grid, {ks} steps",
        }
    line = {
        "metric": "CG step GFLOP/s ((2*nnz + 10n) per step / t) with achieved HBM GB/s",
        "value": round(world * step_flops / (ms * 1e-3) / 1e9, 3),
        "unit": "GFLOP/s",
        "n_gpus": world,
        "steps": res["iterations"],
        "warmup": max(args.warmup, 300),
        "ms_per_step": round(ms, 5),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": args.dtype,
        "data": "synthetic",
        "config": {
            "workload": f"CG on the 7-point Dirichlet Laplacian 256x256x{256 * world} ({N:,} rows, SPD, exact values), rtol 0, {K} steps",
            "nnz": int(nnz_local * world),
            "mrows": info["mrows"],
            "kernel_variant": VNAME[info["variant"]],
            "check_every": check,
            "parallelism": f"row-partitioned x{world}" + (f", {transport} halo + allreduce" if world > 1 else "") + (", ranks share cuda:0 (functional only)" if args.share_gpu else ""),
            "l2": f"inputs larger than L2 ({step_bytes / 1e9:.2f} GB per step); no flush",
        },
        "roofline": {
            "bound": "hbm",
            "kernel": "cg step (SpMV + vector kernels, one CUDA graph per batch)",
            "achieved": round(achieved, 1),
            "peak": peak,
            "peak_source": peak_src,
            "unit": "GB/s",
            "frac": round(achieved / peak, 4),
            "traffic": None,
            "algorithmic_bytes_per_step": int(step_bytes),
        },
        "cpu_baseline": cpu,
        "e2e": {
            "value": round(world * step_flops * r2["iterations"] / te / 1e9, 3),
            "unit": "GFLOP/s",
            "h2d_bytes_per_step": int(N * es),
            "d2h_bytes_per_step": int(N * es),
            "per": f"one solve of {K} steps: H2D b, crsd_cg, D2H x",
            "ms_per_solve": round(te * 1e3, 3),
        },
        "gpu_launches": int(res["launches"]),
        "clocks": clk,
    }
    print(json.dumps(line), flush=True)
    if comm is not None:
        comm.close()
    if world > 1:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def relaunch(args):
    """N > 1 without a torchrun environment: start N ranks ourselves."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
    env = dict(os.environ, OMP_NUM_THREADS=os.environ.get("OMP_NUM_THREADS", str(max(1, host_cores() // args.gpus))))
    return subprocess.call(cmd, env=env)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--config", default="c5", choices=["c1", "c2", "c3", "c3ns", "c4", "c5"])
    ap.add_argument("--dtype", default=None, choices=["f64", "f32"], help="default: f64 (f32 for c4)")
    ap.add_argument("--mrows", type=int, default=0)
    ap.add_argument("--variant", default="auto", choices=list(VARIANTS))
    ap.add_argument("--tune", type=lambda v: int(v, 0), default=0, help="--workload cg: opts.tune of the handle (CRSD_TUNE_*; A/B only)")
    ap.add_argument("--impl", default="crsd", choices=["crsd", "reference"])
    ap.add_argument("--workload", default="spmv", choices=["spmv", "cg"], help="cg: K steps of crsd_cg (N>1: row-partitioned, halo + allreduce)")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-sub", action="store_true", help="N=1 C5: skip the C3 f64/f32 sub-records")
    ap.add_argument("--transport", default="auto", choices=["auto", "nccl", "p2p"], help="N>1 halo exchange: the library's peer-memory kernels (p2p), NCCL send/recv, or auto (p2p if every rank can map its peers, else NCCL)")
    ap.add_argument("--share-gpu", action="store_true", help="N>1 ranks all on cuda:0 (functional check only; needs --transport p2p)")
    args = ap.parse_args()
    if args.dtype is None:
        args.dtype = "f32" if args.config == "c4" else "f64"
    if args.warmup < 3:
        args.warmup = 3
    if args.gpus == 1 or args.impl == "reference":
        # the CPU baseline's OpenMP threads spread over the host cores (read
        # by libgomp at load, i.e. before any OpenMP code runs); not with
        # several ranks per host, whose builders would share the same cores
        os.environ.setdefault("OMP_PROC_BIND", "spread")
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl != "reference":
        sys.exit(relaunch(args))
    if args.impl == "reference":
        run_reference(args)
    elif args.workload == "cg":
        run_cg(args)
    else:
        run_spmv(args)


if __name__ == "__main__":
    main()
