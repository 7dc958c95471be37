#!/usr/bin/env python
"""Benchmark of the CRSD SpMV hot path on B200 (driver contract: one JSON line).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2|c3|c4]
                    [--dtype f64|f32] [--impl crsd|reference]

A step is one y = A*x (alpha 1, beta 0, the paper's SpMV) over the
whole workload, inputs resident in HBM. Workload at N=1: BASELINE.json
configs[1] (C2, 3D 7-point Laplacian 256^3, fp64) unless --config says
otherwise. N>1 (torchrun): weak scaling, rank r owns a 256^3 slab of a
256 x 256 x (256 N) 7-point grid; x halos move with NCCL send/recv over
NVLink inside crsd_spmv_dist, overlapped with the interior segments.

Metric (BASELINE.json): CRSD SpMV GFLOP/s (= 2 nnz / t, whole job) with
achieved HBM GB/s on algorithmic ("unique") bytes and its fraction of the
measured B200 copy bandwidth (MEASURED_PEAKS.json).
--impl reference times the oracle (oracle/coo_spmv.c, long double, 1 thread)
on the host cores on the same workload (the tier's reference arm).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

L2_BYTES = 126 * 1024 * 1024


def _env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            j = json.load(f)
        return float(j.get("hbm_gbs", 6650.0)), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ---------------------------------------------------------------- workloads
def workload(cfg: str, dtype: str, world: int = 1, rank: int = 0):
    """Returns (COO of this rank's rows, description dict, row range or None, global nrows)."""
    import gen

    dt = np.float64 if dtype == "f64" else np.float32
    if cfg == "c1":
        if world != 1:
            raise SystemExit("config c1 is a single-GPU latency workload")
        a = gen.config1()
        N, rb, re = a.nrows, 0, a.nrows
        desc = f"C1: 2D 5-point Laplacian 64x64 ({N:,} rows) + 16 scatter points, {dtype} (L2-resident: latency, L2 flushed before every step)"
    elif cfg == "c2":
        n = 256
        nz = n * world
        N = n * n * nz
        rb, re = rank * n * n * n, (rank + 1) * n * n * n
        a = gen.stencil((n, n, nz), "7pt", values="random", seed=2, row_begin=rb, row_end=re)
        desc = f"C2: 3D 7-point FDM Laplacian 256^3 per GPU (grid 256x256x{nz}, {N:,} rows), {dtype}"
    elif cfg in ("c3", "c3ns"):
        if world != 1:
            raise SystemExit("config c3 is a single-GPU workload")
        # c3ns: the same matrix without its scatter points (diagnostic only)
        a = gen.config3(scatter_frac=0.001 if cfg == "c3" else 0.0)
        N, rb, re = a.nrows, 0, a.nrows
        desc = f"C3: 3D 27-point FVM stencil 192^3 with idle sub-blocks and 0.1% scatter points ({N:,} rows), {dtype}"
    elif cfg == "c5":
        # N > 1: each rank builds its row block of C5 (strong scaling; N = 1 runs run_c5)
        from paper_conf_icpp_sunzwzyr11_b200 import partition_rows

        nn = 768
        N = nn**3
        bounds = partition_rows(N, 256, world)
        rb, re = int(bounds[rank]), int(bounds[rank + 1])
        a = gen.config5(n=nn, values="exact", row_begin=rb, row_end=re)
        desc = f"C5: 3D 7-point Laplacian 768^3 ({N:,} rows), fp64, row-partitioned"
    elif cfg == "c4":
        n = 100_000_000
        if world == 1:
            bounds = np.array([0, n], np.int64)
        else:
            # byte-balanced row blocks (equal rows give
            # max/avg 1.52 on C4): weight per row = its stored diagonals + x + y
            from paper_conf_icpp_sunzwzyr11_b200 import partition_rows

            w = np.empty(n, np.float64)
            for r0, r1, offs in gen.matrices.c4_ranges(n):
                w[r0:r1] = len(offs) + 2
            bounds = partition_rows(n, 512, world, w)
            del w
        rb, re = int(bounds[rank]), int(bounds[rank + 1])
        a = gen.config4(n=n, row_begin=rb, row_end=re)
        N = n
        desc = f"C4: banded, 19 offsets in 9 groups / 4 patterns, 100M rows, {dtype}"
    else:
        raise SystemExit(f"unknown config {cfg}")
    a = gen.COO(N, N, a.row, a.col, a.val.astype(dt))
    return a, desc, (rb, re), N


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
        except Exception:
            self.proc = None

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
        return {
            "sm_mhz": statistics.median(sm) if sm else None,
            "sm_max_mhz": max(mx) if mx else None,
            "reasons": sorted(reasons),
            "samples": len(self.samples),
        }


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


def sustained_copy_bandwidth(dev, seconds):
    """Copy bandwidth sustained over about as long as the timed region
    (back-to-back 1 Gi bf16 copies): the power-capped counterpart of the
    burst figure in MEASURED_PEAKS.json."""
    import torch

    a = torch.empty(1 << 30, dtype=torch.bfloat16, device=f"cuda:{dev}")
    b = torch.empty_like(a)
    b.copy_(a)
    torch.cuda.synchronize()
    n = 0
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    s.record()
    while True:
        for _ in range(10):
            b.copy_(a)
        n += 10
        torch.cuda.synchronize()
        if time.perf_counter() - t0 >= max(seconds, 0.05):
            break
    e.record()
    e.synchronize()
    gbs = n * 2 * a.numel() * 2 / (s.elapsed_time(e) * 1e-3) / 1e9
    del a, b
    torch.cuda.empty_cache()
    return round(gbs, 1)


def load_traffic(cfg, dtype, kernel):
    """ncu dram bytes (read + write) per launch of `kernel` on this workload,
    from one `ncu --set full` capture (profiles/traffic.json, keyed
    "<config>_<dtype>_<kernel>"); None when that kernel was not captured."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            j = json.load(f)
        return j.get(f"{cfg}_{dtype}_{kernel}")
    return None


# ---------------------------------------------------------------- reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle import coo as oracle_coo

    a, desc, _, N = workload(args.config, args.dtype, 1, 0)
    dt = a.val.dtype
    x = np.random.default_rng(7).uniform(-1, 1, a.ncols).astype(dt)
    # bounded sample: calibrate the oracle's rate, then size each step so the
    # whole --steps/--warmup run stays within ~2 minutes of CPU time
    n0, r0_, c0_, v0_ = row_sample(a, 2_000_000)
    t0 = time.perf_counter()
    oracle_coo.coo_spmv(n0, a.ncols, r0_, c0_, v0_, x)
    rate = r0_.shape[0] / max(time.perf_counter() - t0, 1e-6)
    budget = float(os.environ.get("CRSD_REF_BUDGET_S", "120"))
    cap = int(min(a.nnz, max(1_000_000, rate * budget / (args.steps + args.warmup))))
    sample_rows, row, col, val = row_sample(a, cap)
    nnz_s = row.shape[0]
    for _ in range(args.warmup):
        oracle_coo.coo_spmv(sample_rows, a.ncols, row, col, val, x)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle_coo.coo_spmv(sample_rows, a.ncols, row, col, val, x)
        ts.append(time.perf_counter() - t0)
    t = sum(ts) / len(ts)
    gflops = 2.0 * nnz_s / t / 1e9
    sample = f"rows [0,{sample_rows:,}) of the workload, {nnz_s:,} nonzeros per step ({nnz_s / a.nnz:.1%} of the matrix)"
    line = {
        "impl": "reference",
        "metric": "CRSD SpMV GFLOP/s (2*nnz/t)",
        "value": round(gflops, 4),
        "unit": "GFLOP/s",
        "n_gpus": args.gpus,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(t * 1e3, 3),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "f64" if dt == np.float64 else "f32",
        "data": "synthetic",
        "config": {"workload": desc, "alpha": 1.0, "beta": 0.0},
        "cpu_baseline": {"value": round(gflops, 4), "unit": "GFLOP/s", "cores": 1, "kind": "oracle", "sample": sample},
        "e2e": {"value": round(gflops, 4), "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def row_sample(a, cap=None):
    """Rows [0, cut) of the workload, sized to ~cap nonzeros (bounded CPU
    work); entries selected by mask, so input order is irrelevant."""
    if cap is None:
        cap = int(os.environ.get("CRSD_REF_SAMPLE_NNZ", "60000000"))
    if a.nnz <= cap:
        return a.nrows, a.row, a.col, a.val
    cut = max(1, int(a.nrows * cap // a.nnz))
    m = a.row < cut
    return cut, a.row[m], a.col[m], a.val[m]


# ---------------------------------------------------------------- CRSD arm
def cpu_baseline(a, seconds_target=10.0):
    """The oracle as it stands (1 thread, long double) on a bounded row sample."""
    from oracle import coo as oracle_coo

    dt = a.val.dtype
    x = np.random.default_rng(7).uniform(-1, 1, a.ncols).astype(dt)
    nr, row, col, val = row_sample(a)
    k = row.shape[0]
    ts = []
    t_start = time.perf_counter()
    while True:
        t0 = time.perf_counter()
        oracle_coo.coo_spmv(nr, a.ncols, row, col, val, x)
        ts.append(time.perf_counter() - t0)
        if time.perf_counter() - t_start > seconds_target or len(ts) >= 20:
            break
    t = statistics.median(ts)
    return {
        "value": round(2.0 * k / t / 1e9, 4),
        "unit": "GFLOP/s",
        "cores": 1,
        "kind": "oracle",
        "sample": f"rows [0,{nr:,}) ({k:,} nonzeros, {k / a.nnz:.1%} of the workload), median of {len(ts)} runs, long-double accumulation, 1 thread",
    }


def run_crsd(args):
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, Comm, P2PComm

    world = args.gpus
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    # --share-gpu: every rank on cuda:0 (functional check of the multi-rank
    # path on a one-GPU box; NCCL refuses two ranks per GPU, so the torch
    # plumbing uses gloo and the transport must be p2p). Not a scaling number.
    if args.share_gpu:
        local_rank = 0
        if args.transport == "nccl":
            raise SystemExit("--share-gpu needs the p2p transport")
    if world > 1:
        dist.init_process_group("gloo" if args.share_gpu else "nccl", init_method="env://")
        world = dist.get_world_size()
        rank = dist.get_rank()
    torch.cuda.set_device(local_rank)
    dev = local_rank
    red_dev = "cpu" if args.share_gpu else f"cuda:{dev}"

    a, desc, (rb, re), N = workload(args.config, args.dtype, world, rank)
    dt = a.val.dtype
    tdt = torch.float64 if dt == np.float64 else torch.float32
    es = np.dtype(dt).itemsize
    kw = dict(device=dev)
    if args.mrows:
        kw["mrows"] = args.mrows
    kw["variant"] = {"auto": 0, "ldg": 1, "tma": 2, "pipe": 3, "jit": 4}[args.variant]
    if world > 1:
        kw["row_range"] = (rb, re)
    t0 = time.perf_counter()
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, **kw)
    build_s = time.perf_counter() - t0
    info = A.info()
    nnz_local = info["nnz"]
    ub = info["unique_bytes_beta0"]
    stream = torch.cuda.current_stream()

    transport = None
    x_full = torch.from_numpy(np.random.default_rng(7 + rank).uniform(-1, 1, re - rb).astype(dt)).to(f"cuda:{dev}")
    comm = None
    if world > 1:
        lo, nloc, hi = A.x_layout()
        xp = torch.zeros(lo + nloc + hi, dtype=tdt, device=f"cuda:{dev}")
        xp[lo : lo + nloc] = x_full
        y = torch.empty(nloc, dtype=tdt, device=f"cuda:{dev}")
        comm = None
        if args.transport in ("auto", "p2p"):
            try:
                comm = P2PComm(rank, world, dev, mailbox_bytes=max(1 << 20, 4 * (lo + hi) * es))
                transport = "p2p"
            except Exception as e:  # collective: every rank lands here together
                if args.transport == "p2p":
                    raise
                print(f"[bench] peer-memory transport unavailable ({e}); using NCCL", file=sys.stderr)
        if comm is None:
            comm = Comm(rank, world, dev)
            transport = "nccl"
        A.dist_bind(comm)

        def step():
            A.spmv_dist(xp, y, 1.0, 0.0, comm)
    else:
        x = x_full
        y = torch.empty(a.nrows, dtype=tdt, device=f"cuda:{dev}")

        def step():
            A.spmv(x, y, 1.0, 0.0)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if comm is not None and comm.error():
        raise SystemExit(f"[bench] rank {rank}: a peer-memory wait timed out during warm-up (code {comm.error()}); no valid number")

    # timed region: K steps, per-step CUDA events on the launching stream
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    clocks = ClockSampler(dev)
    if not os.environ.get("CRSD_BENCH_NO_CLOCKS"):  # diagnostic switch only
        clocks.start()
        time.sleep(0.3)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_all0 = torch.cuda.Event(enable_timing=True)
    t_all1 = torch.cuda.Event(enable_timing=True)
    t_all0.record(stream)
    launches = 0
    # C1 fits in L2 (0.23 MB): flush it (write a buffer > L2) before every
    # step, outside the step's events; the metric is then the per-step time
    flush = torch.empty(2 * L2_BYTES // 4, dtype=torch.int32, device=f"cuda:{dev}") if args.config == "c1" else None
    for i in range(args.steps):
        if flush is not None:
            flush.zero_()
        ev[i][0].record(stream)
        step()
        ev[i][1].record(stream)
        launches += A.last_launch_count()
    t_all1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    if comm is not None and comm.error():
        raise SystemExit(f"[bench] rank {rank}: a peer-memory wait timed out in the timed region (code {comm.error()}); no valid number")
    total_ms = t_all0.elapsed_time(t_all1)
    step_ms = [s.elapsed_time(e) for s, e in ev]
    if world > 1:
        tt = torch.tensor([total_ms], dtype=torch.float64, device=red_dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        total_ms = float(tt.item())
        nn = torch.tensor([nnz_local, ub], dtype=torch.float64, device=red_dev)
        dist.all_reduce(nn)
        nnz_all, ub_all = float(nn[0].item()), float(nn[1].item())
    else:
        nnz_all, ub_all = float(nnz_local), float(ub)
    ms = total_ms / args.steps
    if flush is not None:
        ms = statistics.median(step_ms)
    gflops = 2.0 * nnz_all / (ms * 1e-3) / 1e9
    kern_ms = statistics.mean(step_ms)
    peak, peak_src = measured_peaks()
    achieved = ub / (kern_ms * 1e-3) / 1e9

    # e2e through the public C-ABI with host buffers (pinned), N = 1 path
    e2e = None
    if world == 1:
        xh = torch.from_numpy(np.random.default_rng(7).uniform(-1, 1, a.ncols).astype(dt)).pin_memory()
        yh = torch.empty(a.nrows, dtype=tdt).pin_memory()
        for _ in range(2):
            A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr(), 1.0, 0.0)
        ke = max(3, min(args.steps, 50))
        t0 = time.perf_counter()
        for _ in range(ke):
            A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr(), 1.0, 0.0)
        te = (time.perf_counter() - t0) / ke
        # transfer bound of the e2e step: pinned H2D / D2H bandwidth alone
        xd_tmp = torch.empty(a.ncols, dtype=tdt, device=f"cuda:{dev}")
        yd_tmp = torch.empty(a.nrows, dtype=tdt, device=f"cuda:{dev}")

        def bw(fn, nbytes):
            fn()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            for _ in range(5):
                fn()
            torch.cuda.synchronize()
            return nbytes * 5 / (time.perf_counter() - t0) / 1e9

        h2d = bw(lambda: xd_tmp.copy_(xh, non_blocking=True), a.ncols * es)
        d2h = bw(lambda: yh.copy_(yd_tmp, non_blocking=True), a.nrows * es)
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

        def both():  # H2D and D2H at the same time on two streams
            with torch.cuda.stream(s1):
                xd_tmp.copy_(xh, non_blocking=True)
            with torch.cuda.stream(s2):
                yh.copy_(yd_tmp, non_blocking=True)

        bidir_ms = bw(both, 1e6) and None
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(5):
            both()
        torch.cuda.synchronize()
        bidir_ms = (time.perf_counter() - t0) / 5 * 1e3
        del xd_tmp, yd_tmp
        e2e = {
            "value": round(2.0 * nnz_all / te / 1e9, 3),
            "unit": "GFLOP/s",
            "h2d_bytes_per_step": int(a.ncols * es),
            "d2h_bytes_per_step": int(a.nrows * es),
            "ms_per_step": round(te * 1e3, 4),
            "pinned_h2d_gbs": round(h2d, 1),
            "pinned_d2h_gbs": round(d2h, 1),
            "transfer_bound_ms": round(max(a.ncols * es / h2d, a.nrows * es / d2h) / 1e6, 4),
            "concurrent_h2d_d2h_ms": round(bidir_ms, 4),
            "path": "crsd_spmv_host: chunked H2D(x) / kernel / D2H(y) pipeline on three streams",
        }
    if world > 1:
        # e2e through crsd_spmv_dist: pinned host x slice -> owned part of
        # x_padded, halo exchange + SpMV, y slice -> pinned host; max over ranks
        xh = torch.from_numpy(np.random.default_rng(7 + rank).uniform(-1, 1, re - rb).astype(dt)).pin_memory()
        yh = torch.empty(re - rb, dtype=tdt).pin_memory()

        def e2e_step():
            xp[lo : lo + nloc].copy_(xh, non_blocking=True)
            A.spmv_dist(xp, y, 1.0, 0.0, comm)
            yh.copy_(y, non_blocking=True)
            torch.cuda.current_stream().synchronize()

        for _ in range(2):
            e2e_step()
        ke = max(3, min(args.steps, 50))
        dist.barrier()
        t0 = time.perf_counter()
        for _ in range(ke):
            e2e_step()
        te = torch.tensor([(time.perf_counter() - t0) / ke], dtype=torch.float64, device=red_dev)
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
        te = float(te.item())
        e2e = {
            "value": round(2.0 * nnz_all / te / 1e9, 3),
            "unit": "GFLOP/s",
            "h2d_bytes_per_step": int((re - rb) * es) * world,
            "d2h_bytes_per_step": int((re - rb) * es) * world,
            "ms_per_step": round(te * 1e3, 4),
            "path": f"per rank: H2D of the owned x slice, crsd_spmv_dist ({transport} halo + SpMV), D2H of the y slice; max over ranks",
        }
    if rank != 0:
        if comm is not None:
            comm.close()
        dist.destroy_process_group()
        return

    cpu = None if (world > 1 or args.no_cpu) else cpu_baseline(a)
    box_copy = copy_bandwidth(dev)
    box_copy_sus = sustained_copy_bandwidth(dev, total_ms * 1e-3)
    kname = {1: "crsd_spmv_ldg", 2: "crsd_spmv_tma", 3: "crsd_spmv_pipe", 4: "crsd_jit"}[info["variant"]]
    traffic = None if args.mrows else load_traffic(args.config, args.dtype, kname)
    line = {
        "metric": "CRSD SpMV GFLOP/s (2*nnz/t) with achieved HBM GB/s (% of B200 peak)",
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
            "mrows": info["mrows"],
            "kernel_variant": {1: "ldg", 2: "tma", 3: "pipe", 4: "jit"}[info["variant"]],
            "alpha": 1.0,
            "beta": 0.0,
            "patterns": info["npat"],
            "instances": info["ninst"],
            "fills": info["nfills"],
            "scatter": info["nscatter"],
            "l2": (f"inputs larger than L2 ({ub / 1e9:.2f} GB streamed per step vs {L2_BYTES / 2**20:.0f} MiB L2); no flush" if flush is None else f"L2 flushed (252 MiB written) before every step; ms_per_step = median per-step CUDA-event time"),
            "build_s": round(build_s, 2),
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
            "traffic": traffic,
            "algorithmic_bytes_per_launch": int(ub),
            "avg_launch_ms": round(kern_ms, 5),
            "launches_per_step": round(launches / max(1, args.steps), 2),
            "per_step_note": "with several launches per step (JIT occupancy classes, dist interior/boundary) achieved = the step's algorithmic bytes / the step's CUDA-event time",
            "copy_gbs_this_box": box_copy,
            "frac_of_this_box_copy": round(achieved / box_copy, 4) if box_copy else None,
            "sustained_copy_gbs_this_box": box_copy_sus,
            "sustained_copy_note": "copies for as long as the timed region; long runs hit the 1 kW power cap",
        },
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": int(launches),
        "clocks": clk,
    }
    print(json.dumps(line), flush=True)
    if comm is not None:
        comm.close()
    if world > 1:
        dist.destroy_process_group()


# ---------------------------------------------------------------- C5 on one GPU
def run_c5(args):
    """--config c5: BASELINE config 5 (3D 7-point Laplacian 768^3, fp64,
    452,984,832 rows, 3.17e9 nonzeros, 32.6 GB) on ONE B200. The host builds
    it as 8 row blocks (the 8-GPU partition: a single 3.17e9-entry COO would
    need ~76 GB of host RAM plus the builder's copies), every block resident
    on the GPU; the blocks share one global x (each block's padded x is a
    view of it: its halos are the neighbours' owned x, no exchange) and write
    disjoint slices of one global y. A step = the 8 blocks' crsd_spmv_dist
    calls (comm = NULL)."""
    import torch

    import gen
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, partition_rows

    if args.gpus != 1:
        raise SystemExit("run_c5 is the one-GPU form")
    if args.dtype != "f64":
        raise SystemExit("config c5 is fp64")
    torch.cuda.set_device(0)
    nn, nb = 768, 8
    N = nn**3
    bounds = partition_rows(N, 256, nb)
    blocks, t0 = [], time.perf_counter()
    cpu = None
    for k in range(nb):
        rb, re = int(bounds[k]), int(bounds[k + 1])
        a = gen.config5(n=nn, values="exact", row_begin=rb, row_end=re)
        if k == 0 and not args.no_cpu:
            cpu = cpu_baseline(gen.COO(re, N, a.row, a.col, a.val))
            cpu["sample"] += " (block 0 of the 8 host-built blocks)"
        A = CRSDMatrix.from_coo(N, N, a.row, a.col, a.val, row_range=(rb, re), device=0)
        del a
        blocks.append((rb, re, A))
    build_s = time.perf_counter() - t0
    pad = (max(max(A.x_layout()[0], A.x_layout()[2]) for _, _, A in blocks) + 64 + 3) // 4 * 4  # keeps views 16-B aligned
    x_ext = torch.zeros(N + 2 * pad, dtype=torch.float64, device="cuda:0")
    x = x_ext[pad : pad + N]
    x.copy_(torch.from_numpy(np.random.default_rng(7).uniform(-1, 1, N)))
    y = torch.empty(N, dtype=torch.float64, device="cuda:0")
    views = []
    for rb, re, A in blocks:
        lo, nloc, hi = A.x_layout()
        views.append((A, x_ext[pad + rb - lo : pad + re + hi], y[rb:re]))
    infos = [A.info() for _, _, A in blocks]
    nnz = sum(i["nnz"] for i in infos)
    ub = sum(i["unique_bytes_beta0"] for i in infos)

    def step():
        for A, xv, yv in views:
            A.spmv_dist(xv, yv, 1.0, 0.0, None)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    clocks = ClockSampler(0)
    clocks.start()
    time.sleep(0.3)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    launches = 0
    torch.cuda.synchronize()
    for i in range(args.steps):
        ev[i][0].record(stream)
        step()
        ev[i][1].record(stream)
        launches += sum(A.last_launch_count() for A, _, _ in views)
    torch.cuda.synchronize()
    clk = clocks.stop()
    step_ms = [s_.elapsed_time(e_) for s_, e_ in ev]
    ms = statistics.mean(step_ms)
    peak, peak_src = measured_peaks()
    achieved = ub / (ms * 1e-3) / 1e9
    # e2e: pinned host x -> device, the 8 block SpMVs, device y -> pinned host
    xh = torch.from_numpy(np.random.default_rng(7).uniform(-1, 1, N)).pin_memory()
    yh = torch.empty(N, dtype=torch.float64).pin_memory()

    def e2e_step():
        x.copy_(xh, non_blocking=True)
        step()
        yh.copy_(y, non_blocking=True)
        torch.cuda.synchronize()

    e2e_step()
    ke = 5
    t0 = time.perf_counter()
    for _ in range(ke):
        e2e_step()
    te = (time.perf_counter() - t0) / ke
    line = {
        "metric": "CRSD SpMV GFLOP/s (2*nnz/t) with achieved HBM GB/s (% of B200 peak)",
        "value": round(2.0 * nnz / (ms * 1e-3) / 1e9, 3),
        "unit": "GFLOP/s",
        "n_gpus": 1,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(ms, 5),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "f64",
        "data": "synthetic",
        "config": {
            "workload": f"C5: 3D 7-point Laplacian 768^3 ({N:,} rows), fp64, one B200, 8 resident row blocks sharing one x",
            "nnz": int(nnz),
            "mrows": infos[0]["mrows"],
            "kernel_variant": {1: "ldg", 2: "tma", 3: "pipe", 4: "jit"}[infos[0]["variant"]],
            "alpha": 1.0,
            "beta": 0.0,
            "device_bytes": int(sum(i["device_bytes"] for i in infos) + (N + 2 * pad + N) * 8),
            "l2": f"inputs larger than L2 ({ub / 1e9:.1f} GB per step); no flush",
            "build_s": round(build_s, 1),
            "parallelism": "one GPU",
        },
        "hbm_gbs": round(achieved, 1),
        "hbm_frac_of_peak": round(achieved / peak, 4),
        "roofline": {
            "bound": "hbm",
            "kernel": "crsd_jit (8 blocks x interior range + boundary list per step)",
            "achieved": round(achieved, 1),
            "peak": peak,
            "peak_source": peak_src,
            "unit": "GB/s",
            "frac": round(achieved / peak, 4),
            "traffic": None,
            "algorithmic_bytes_per_step": int(ub),
            "avg_step_ms": round(ms, 5),
            "launches_per_step": round(launches / max(1, args.steps), 2),
        },
        "cpu_baseline": cpu,
        "e2e": {
            "value": round(2.0 * nnz / te / 1e9, 3),
            "unit": "GFLOP/s",
            "h2d_bytes_per_step": int(N * 8),
            "d2h_bytes_per_step": int(N * 8),
            "ms_per_step": round(te * 1e3, 3),
            "path": "pinned H2D of x (3.6 GB), the 8 block SpMVs, pinned D2H of y (3.6 GB); serial",
        },
        "gpu_launches": int(launches),
        "clocks": clk,
    }
    print(json.dumps(line), flush=True)


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

    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, Comm, P2PComm
    from oracle import cg_ref

    import gen

    world = args.gpus
    rank = int(os.environ.get("RANK", "0"))
    local_rank = 0 if args.share_gpu else int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        dist.init_process_group("gloo" if args.share_gpu else "nccl", init_method="env://")
        world, rank = dist.get_world_size(), dist.get_rank()
    torch.cuda.set_device(local_rank)
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
    A = CRSDMatrix.from_coo(N, N, a.row, a.col, a.val, device=local_rank, **kw)
    info = A.info()
    comm, transport = None, None
    if world > 1:
        lo, _, hi = A.x_layout()
        if args.transport in ("auto", "p2p"):
            try:
                comm, transport = P2PComm(rank, world, local_rank, mailbox_bytes=max(1 << 20, 4 * (lo + hi) * es)), "p2p"
            except Exception as e:
                if args.transport == "p2p":
                    raise
                print(f"[bench] peer-memory transport unavailable ({e}); using NCCL", file=sys.stderr)
        if comm is None:
            comm, transport = Comm(rank, world, local_rank), "nccl"
        A.dist_bind(comm)
    vec_passes = 10
    step_bytes = info["unique_bytes_beta0"] + vec_passes * nloc * es
    nnz_local = int(a.nnz)
    step_flops = 2.0 * nnz_local + 10.0 * nloc
    rng = np.random.default_rng(17 + rank)
    bh = torch.from_numpy(rng.uniform(-1, 1, nloc).astype(dt)).pin_memory()
    b = bh.to(dev)
    x = torch.zeros(nloc, dtype=tdt, device=dev)
    K = args.steps
    check = min(K, 50)
    clocks = ClockSampler(local_rank)
    clocks.start()
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
    if world == 1:
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
            "kernel_variant": {1: "ldg", 2: "tma", 3: "pipe", 4: "jit"}[info["variant"]],
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--config", default="c2", choices=["c1", "c2", "c3", "c3ns", "c4", "c5"])
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--mrows", type=int, default=0)
    ap.add_argument("--variant", default="auto", choices=["auto", "ldg", "tma", "pipe", "jit"])
    ap.add_argument("--impl", default="crsd", choices=["crsd", "reference"])
    ap.add_argument("--workload", default="spmv", choices=["spmv", "cg"], help="cg: K steps of crsd_cg (N>1: row-partitioned, halo + allreduce)")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--transport", default="auto", choices=["auto", "nccl", "p2p"], help="N>1 halo exchange: the library's peer-memory kernels (p2p), NCCL send/recv, or auto (p2p if every rank can map its peers, else NCCL)")
    ap.add_argument("--share-gpu", action="store_true", help="N>1 ranks all on cuda:0 (functional check only; needs --transport p2p)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    elif args.workload == "cg":
        run_cg(args)
    elif args.config == "c5" and args.gpus == 1:
        run_c5(args)
    else:
        run_crsd(args)


if __name__ == "__main__":
    main()
