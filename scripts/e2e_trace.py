#!/usr/bin/env python
"""Timeline of crsd_spmv_host (the e2e path): a CUPTI trace (torch.profiler)
of a few calls, summarised per call: span, H2D busy time and span, D2H busy
time and span, kernel time, and the gaps -- where the pipeline is not
transfer-bound.

usage: python scripts/e2e_trace.py [c2|c5] [chunks (0: the library's default)]
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
    chunks = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    torch.cuda.set_device(0)
    from gen import fast
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix

    n1 = {"c2": 256, "c5": 768}[cfg]
    d = (n1, n1, n1)
    N = n1**3
    ptr, col, val = fast.stencil(d, bench._stencil_disps("7pt", d), False, cfg == "c2", 2, None, 0, N, csr=True)
    A = CRSDMatrix.from_csr(N, N, ptr, col, val, device=0, e2e_chunks=chunks)
    del ptr, col, val
    xh = torch.from_numpy(np.random.default_rng(7).uniform(-1, 1, N)).pin_memory()
    yh = torch.empty(N, dtype=torch.float64).pin_memory()
    for _ in range(3):
        A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr(), 1.0, 0.0)
    from torch.profiler import ProfilerActivity, profile

    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for _ in range(3):
            A.spmv_host_ptr(xh.data_ptr(), yh.data_ptr(), 1.0, 0.0)
    out = os.path.join(ROOT, "gpurun_out", "e2e_trace")
    os.makedirs(out, exist_ok=True)
    path = os.path.join(out, f"trace_{cfg}.json")
    prof.export_chrome_trace(path)
    ev = json.load(open(path))["traceEvents"]
    acts = [e for e in ev if e.get("cat") in ("kernel", "gpu_memcpy")]
    acts.sort(key=lambda e: e["ts"])
    # split into calls: a call starts with the first H2D after a D2H-only stretch
    calls, cur, last_kind = [], [], None
    for e in acts:
        kind = "k" if e["cat"] == "kernel" else ("h2d" if "HtoD" in e["name"] else "d2h")
        if kind == "h2d" and last_kind == "d2h" and cur:
            calls.append(cur)
            cur = []
        cur.append((kind, e["ts"], e["ts"] + e["dur"]))
        last_kind = kind
    if cur:
        calls.append(cur)
    for c in calls:
        t0, t1 = min(a for _, a, _ in c), max(b for _, _, b in c)
        summ = {"span_ms": round((t1 - t0) / 1e3, 3)}
        for k in ("h2d", "d2h", "k"):
            xs = [(a, b) for kk, a, b in c if kk == k]
            if xs:
                summ[k] = {"n": len(xs), "busy_ms": round(sum(b - a for a, b in xs) / 1e3, 3),
                           "first_start_ms": round((xs[0][0] - t0) / 1e3, 3), "last_end_ms": round((max(b for _, b in xs) - t0) / 1e3, 3)}
        print(json.dumps({"config": cfg, **summ}), flush=True)


if __name__ == "__main__":
    main()
