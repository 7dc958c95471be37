#!/usr/bin/env python
"""crsd_spmv_host: uniform vs ramped chunks (CRSD_E2E_RAMP), interleaved, C2 fp64 and C3 fp64."""
import os, sys, time
import numpy as np, torch
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix
torch.cuda.set_device(0)
for cfg in ("c2", "c3"):
    a, _, _, _ = bench.workload(cfg, "f64", 1, 0)
    xh = torch.from_numpy(np.random.default_rng(7).uniform(-1, 1, a.ncols)).pin_memory()
    yh = torch.empty(a.nrows, dtype=torch.float64).pin_memory()
    for rep in range(2):
        for ramp in ("0", "1"):
            for ch in ("16", "24", "32"):
                os.environ["CRSD_E2E_RAMP"] = ramp
                os.environ["CRSD_E2E_CHUNKS"] = ch
                A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val)
                for _ in range(3):
                    A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr())
                t0 = time.perf_counter()
                for _ in range(30):
                    A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr())
                print(f"{cfg} rep {rep} ramp {ramp} chunks {ch}: {(time.perf_counter() - t0) / 30 * 1e3:.3f} ms/step", flush=True)
                del A
