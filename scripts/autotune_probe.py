#!/usr/bin/env python
"""crsd_create_autotuned on the BASELINE workloads: which mrows / variant wins
and at what fraction of the measured copy peak (evidence for DESIGN.md §14).
usage: python scripts/autotune_probe.py [c2:f64 c3:f32 ...]"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix  # noqa: E402

PEAK = bench.measured_peaks()[0]
CANDS = {"f64": (128, 256, 512), "f32": (256, 512, 1024)}
for case in sys.argv[1:] or ["c2:f64", "c2:f32", "c3:f64", "c3:f32", "c4:f32"]:
    cfg, dt = case.split(":")
    a = bench.coo_matrix(cfg, dt)
    A, ms = CRSDMatrix.autotuned(a.nrows, a.ncols, a.row, a.col, a.val, mrows_candidates=CANDS[dt], reps=50)
    inf = A.info()
    best = ms[inf["mrows"]]
    print(json.dumps({"case": case, "chosen_mrows": inf["mrows"], "variant": inf["variant"], "ms_per_mrows": ms,
                      "frac": round(inf["unique_bytes_beta0"] / (best * 1e-3) / 1e9 / PEAK, 4)}), flush=True)
    del A, a
