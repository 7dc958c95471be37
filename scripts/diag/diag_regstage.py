"""Register-staging depth diagnostic. NOT a
product path: needs a diagnostic build of libcrsd.so whose reg_diags adds
CRSD_DIAG_REXTRA diagonals to R and whose crsd_jit_rs launch bounds take
CRSD_DIAG_MINB CTAs per SM; with the product build both variables have no
effect.

usage: python scripts/diag/diag_regstage.py c3:f64
"""
import json, os, sys
import torch
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import bench
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix
PEAK = bench.measured_peaks()[0]
SET = [("def", None, None), ("x2b4", "2", "4"), ("x4b4", "4", "4"), ("x6b4", "6", "4"), ("x0b4", "0", "4")]
def t(A, x, y, steps=200):
    for _ in range(10): A.spmv(x, y)
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(steps): A.spmv(x, y)
    e.record(); e.synchronize()
    return s.elapsed_time(e) / steps
for case in sys.argv[1:]:
    cfg, dt = case.split(":")[:2]
    a = bench.coo_matrix(cfg, dt)
    tdt = torch.float64 if dt == "f64" else torch.float32
    x = torch.rand(a.ncols, dtype=tdt, device="cuda"); y = torch.empty(a.nrows, dtype=tdt, device="cuda")
    mats = []
    for name, rx, mb in SET:
        for k, v in (("CRSD_DIAG_REXTRA", rx), ("CRSD_DIAG_MINB", mb)):
            if v is None: os.environ.pop(k, None)
            else: os.environ[k] = v
        mats.append((name, CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, variant=4)))
    ub = mats[0][1].info()["unique_bytes_beta0"]
    for rep in range(4):
        for name, A in mats:
            ms = t(A, x, y)
            print(json.dumps({"case": case, "setting": name, "rep": rep, "ms": round(ms, 5), "frac": round(ub / (ms * 1e-3) / 1e9 / PEAK, 4), "launches": A.last_launch_count()}), flush=True)
