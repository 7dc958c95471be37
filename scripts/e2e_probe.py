#!/usr/bin/env python
"""crsd_spmv_host chunk-count probe (C2 fp64): ms per end-to-end step."""
import os, sys, time
import numpy as np, torch
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix
torch.cuda.set_device(0)
a = bench.coo_matrix("c2", "f64")
xh = torch.from_numpy(np.random.default_rng(7).uniform(-1, 1, a.ncols)).pin_memory()
yh = torch.empty(a.nrows, dtype=torch.float64).pin_memory()
for ch in sys.argv[1:] or ["8", "16", "32", "64"]:
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, e2e_chunks=int(ch))
    for _ in range(3):
        A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr())
    t0 = time.perf_counter()
    for _ in range(30):
        A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr())
    print(f"chunks {ch}: {(time.perf_counter() - t0) / 30 * 1e3:.3f} ms/step, launches {A.last_launch_count()}", flush=True)
    del A
