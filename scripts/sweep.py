#!/usr/bin/env python
"""JIT codelet A/B sweep on one GPU (tuning evidence for DESIGN.md).

Generates each workload once, builds one handle per setting and times
crsd_spmv (y = A x) for each, interleaved over REPS rounds so box drift hits
every setting alike. Prints one JSON line per (case, setting, round).

usage: python scripts/sweep.py c3:f64 c3:f32:256 ...
  SWEEP_SET  ';'-separated settings "name=chunk,tune[,variant]" (default:
             chunk -1/0/4 with the baked lookup, and 0 with descriptor issue)
  SWEEP_REPS rounds (default 2); SWEEP_STEPS launches per timing (default 200)
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix  # noqa: E402

PEAK = bench.measured_peaks()[0]
DEFAULT_SET = "one=-1,0;win=0,0;k4=4,0;desc=0,1"


def time_it(A, x, y, steps, warm=10):
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
    cases = sys.argv[1:] or ["c2:f64", "c2:f32", "c3:f64", "c3:f32:256"]
    settings = []
    for item in os.environ.get("SWEEP_SET", DEFAULT_SET).split(";"):
        name, vals = item.split("=")
        v = [int(t, 0) for t in vals.split(",")]
        settings.append((name, v[0], v[1], v[2] if len(v) > 2 else 4))
    reps = int(os.environ.get("SWEEP_REPS", "2"))
    steps = int(os.environ.get("SWEEP_STEPS", "200"))
    torch.cuda.set_device(0)
    for case in cases:
        parts = case.split(":")
        cfg, dt = parts[0], parts[1]
        mrows = int(parts[2]) if len(parts) > 2 else 0
        a = bench.coo_matrix(cfg, dt)
        tdt = torch.float64 if dt == "f64" else torch.float32
        x = torch.rand(a.ncols, dtype=tdt, device="cuda")
        y = torch.empty(a.nrows, dtype=tdt, device="cuda")
        mats = []
        for name, chunk, tune, variant in settings:
            try:
                A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, mrows=mrows, variant=variant,
                                        jit_chunk=chunk, tune=tune)
                mats.append((name, chunk, tune, A))
            except Exception as ex:
                print(json.dumps({"case": case, "setting": name, "error": str(ex)[:200]}), flush=True)
        del a
        for rep in range(reps):
            for name, chunk, tune, A in mats:
                inf = A.info()
                ub = inf["unique_bytes_beta0"]
                ms = time_it(A, x, y, steps)
                gbs = ub / (ms * 1e-3) / 1e9
                print(json.dumps({"case": case, "mrows": inf["mrows"], "setting": name, "jit_chunk": chunk, "tune": tune,
                                  "variant": inf["variant"], "rep": rep, "ms": round(ms, 5), "GBps": round(gbs, 1),
                                  "frac": round(gbs / PEAK, 4), "smem": inf["smem_bytes"], "unique_bytes": ub,
                                  "launches": A.last_launch_count()}), flush=True)
        del mats
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
