#!/usr/bin/env python
"""Small runs of every kernel variant for compute-sanitizer (memcheck /
racecheck / synccheck / initcheck). Checks parity too, so a silent race shows
up either as a sanitizer report or as a parity failure.

usage: compute-sanitizer --tool racecheck python scripts/sanitize.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gen  # noqa: E402
from oracle import coo  # noqa: E402
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix  # noqa: E402


def main():
    torch.cuda.set_device(0)
    cases = [("c1", gen.config1()), ("c3s", gen.config3(n=20)), ("band", gen.config4(n=120_000))]
    bad = 0
    for name, a in cases:
        for dt in (np.float64, np.float32):
            b = a.astype(dt)
            x = np.random.default_rng(1).uniform(-1, 1, b.ncols).astype(dt)
            y0 = np.random.default_rng(2).uniform(-1, 1, b.nrows).astype(dt)
            yref, sc = coo.coo_spmv(b.nrows, b.ncols, b.row, b.col, b.val, x, -0.75, 0.5, y0)
            # variants 1-4; the JIT codelet also with one barrier (-1), two
            # diagonals per chunk (2) and descriptor-issued copies (tune 1)
            for v, chunk, tune in ((1, 0, 0), (2, 0, 0), (3, 0, 0), (4, 0, 0), (4, -1, 0), (4, 2, 0), (4, 0, 1)):
                A = CRSDMatrix.from_coo(b.nrows, b.ncols, b.row, b.col, b.val, variant=v, jit_chunk=chunk, tune=tune)
                tdt = torch.float64 if dt == np.float64 else torch.float32
                xd = torch.from_numpy(x).to("cuda", tdt)
                yd = torch.from_numpy(y0).to("cuda", tdt)
                A.spmv(xd, yd, -0.75, 0.5)
                torch.cuda.synchronize()
                err = coo.parity_error(yd.cpu().numpy(), yref, sc)
                ok = err <= (1e-12 if dt == np.float64 else 1e-5)
                bad += not ok
                print(f"{name} {np.dtype(dt).name} variant {v} chunk {chunk} tune {tune}: parity {err:.2e} {'ok' if ok else 'FAIL'}", flush=True)
    # JIT launches split by occupancy class (forced on a small C4: several
    # ranges with their own dynamic smem)
    from paper_conf_icpp_sunzwzyr11_b200 import TUNE_JIT_SPLIT_ALL

    for dt in (np.float64, np.float32):
        b = gen.config4(n=400_000).astype(dt)
        x = np.random.default_rng(1).uniform(-1, 1, b.ncols).astype(dt)
        yref, sc = coo.coo_spmv(b.nrows, b.ncols, b.row, b.col, b.val, x)
        A = CRSDMatrix.from_coo(b.nrows, b.ncols, b.row, b.col, b.val, variant=4, mrows=512, tune=TUNE_JIT_SPLIT_ALL)
        tdt = torch.float64 if dt == np.float64 else torch.float32
        xd = torch.from_numpy(x).to("cuda", tdt)
        yd = torch.full((b.nrows,), float("nan"), device="cuda", dtype=tdt)
        A.spmv(xd, yd)
        torch.cuda.synchronize()
        err = coo.parity_error(yd.cpu().numpy(), yref, sc)
        ok = err <= (1e-12 if dt == np.float64 else 1e-5) and A.last_launch_count() > 1
        bad += not ok
        print(f"c4 ranges {np.dtype(dt).name}: {A.last_launch_count()} launches, parity {err:.2e} {'ok' if ok else 'FAIL'}", flush=True)
    # CG (vector kernels, grid reductions, graph replay) on an SPD stencil
    from oracle import cg_ref

    a = gen.spd_stencil_scatter((12, 12, 12), "7pt", n_pairs=30, seed=2)
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val)
    rng = np.random.default_rng(3)
    b = rng.uniform(-1, 1, a.nrows)
    bd = torch.from_numpy(b).to("cuda")
    xd = torch.zeros(a.nrows, dtype=torch.float64, device="cuda")
    res = A.cg(bd, xd, 20, 0.0, check_every=6, history=True)
    xr, _, hr = cg_ref.cg(a, b, np.zeros(a.nrows), 20)
    ex = np.max(np.abs(xd.cpu().numpy() - xr)) / np.max(np.abs(xr))
    ok = res["iterations"] == 20 and ex <= 1e-12
    bad += not ok
    print(f"cg f64: 20 steps, x deviation {ex:.2e} {'ok' if ok else 'FAIL'}", flush=True)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
