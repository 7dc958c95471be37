#!/usr/bin/env python
"""CG throughput on one GPU (SURVEY.md §8(f) NEXT 2 evidence).

C2 grid (7-point Dirichlet Laplacian, SPD) at n^3, fixed K steps (rtol 0),
timed with CUDA events around crsd_cg (one graph replay per check_every
steps, device-side scalars). Bytes per step: the SpMV's unique bytes plus the
vector traffic of the three vector kernels ((p,q): 2 reads; r update: 2
reads + 1 write; x and p update: 3 reads + 2 writes = 10 vectors).
usage: python scripts/cg_bench.py [n] [K] [f64|f32]
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
K = int(sys.argv[2]) if len(sys.argv) > 2 else 200
dt = np.float64 if (len(sys.argv) <= 3 or sys.argv[3] == "f64") else np.float32
check = int(os.environ.get("CG_CHECK", "50"))
a = gen.spd_stencil_scatter((n, n, n), "7pt").astype(dt)
A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val)
N = a.nrows
tdt = torch.float64 if dt == np.float64 else torch.float32
b = torch.rand(N, dtype=tdt, device="cuda") - 0.5
x = torch.zeros(N, dtype=tdt, device="cuda")
A.cg(b, x, 300, 0.0, check_every=check)  # warm-up (workspace, graph, clocks)
torch.cuda.synchronize()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
x.zero_()
s.record()
res = A.cg(b, x, K, 0.0, check_every=check)
e.record()
e.synchronize()
ms = s.elapsed_time(e)
es = np.dtype(dt).itemsize
inf = A.info()
step_bytes = inf["unique_bytes_beta0"] + 10 * N * es
per = ms / res["iterations"]
print(json.dumps({"workload": f"CG 7-pt {n}^3 {np.dtype(dt).name}", "variant": inf["variant"], "steps": res["iterations"],
                  "ms_per_step": round(per, 5), "GBps": round(step_bytes / (per * 1e-3) / 1e9, 1),
                  "spmv_bytes": inf["unique_bytes_beta0"], "step_bytes": step_bytes,
                  "launches": res["launches"], "rr_ratio": res["rr"] / res["rr0"]}), flush=True)
