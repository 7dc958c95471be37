#!/usr/bin/env python
"""Kernel-variant / pipeline-shape sweep on one GPU (tuning evidence for DESIGN.md).

Generates each workload once, then times crsd_spmv (y = A x) for every
variant and CRSD_PIPE_* shape override. Prints one JSON line per case.
usage: python scripts/sweep.py [c2:f64 c3:f64 ...]
"""
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix  # noqa: E402

PEAK = bench.measured_peaks()[0]
SHAPES = [s for s in os.environ.get("SWEEP_PIPE", "none").split(";") if s]
SHAPES = [None if s == "none" else tuple(int(v) for v in s.split(",")) for s in SHAPES]
TMA = [s for s in os.environ.get("SWEEP_TMA", "none").split(";") if s]
TMA = [None if s == "none" else (s.split("=")[0], int(s.split("=")[1])) for s in TMA]


def time_it(A, x, y, steps=200, warm=10):
    for _ in range(warm):
        A.spmv(x, y)
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(steps):
        A.spmv(x, y)
    e.record()
    e.synchronize()
    return s.elapsed_time(e) / steps


def main():
    cases = sys.argv[1:] or ["c2:f64", "c2:f32", "c3:f64", "c3:f32"]
    torch.cuda.set_device(0)
    for case in cases:
        parts = case.split(":")
        cfg, dt = parts[0], parts[1]
        mrows = int(parts[2]) if len(parts) > 2 else 256
        a, desc, _, _ = bench.workload(cfg, dt, 1, 0)
        tdt = torch.float64 if dt == "f64" else torch.float32
        x = torch.rand(a.ncols, dtype=tdt, device="cuda")
        y = torch.empty(a.nrows, dtype=tdt, device="cuda")
        runs = [("ldg", 1, None)] + [("tma", 2, t) for t in TMA] + [("pipe", 3, sh) for sh in SHAPES] + [("jit", 4, None), ("jit_late", 4, None), ("jitp", 4, None)]
        only = os.environ.get("SWEEP_VARIANTS")
        if only:
            runs = [r for r in runs if r[0] in only.split(",")]
        for name, v, sh in runs:
            for k in ("CRSD_PIPE_PERSM", "CRSD_PIPE_NX", "CRSD_PIPE_NS", "CRSD_TMA_Q", "CRSD_TMA_SPLIT", "CRSD_JIT_EARLY", "CRSD_JIT_MODE"):
                os.environ.pop(k, None)
            if name == "jit_late":
                os.environ["CRSD_JIT_EARLY"] = "0"
            if name == "jitp":
                os.environ["CRSD_JIT_MODE"] = "persist"
            if sh and name == "tma":
                os.environ["CRSD_TMA_" + sh[0]] = str(sh[1])
            elif sh:
                os.environ["CRSD_PIPE_PERSM"], os.environ["CRSD_PIPE_NX"], os.environ["CRSD_PIPE_NS"] = map(str, sh)
            try:
                A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=mrows, variant=v)
            except Exception as ex:
                print(json.dumps({"case": case, "variant": name, "shape": sh, "error": str(ex)[:200]}), flush=True)
                continue
            ub = A.info()["unique_bytes_beta0"]
            ms = time_it(A, x, y)
            gbs = ub / (ms * 1e-3) / 1e9
            print(json.dumps({"case": case, "mrows": mrows, "variant": name, "shape": sh, "ms": round(ms, 5), "GBps": round(gbs, 1), "frac": round(gbs / PEAK, 4), "smem": A.info()["smem_bytes"], "unique_bytes": ub, "launches": A.last_launch_count()}), flush=True)
            del A
        del a
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
