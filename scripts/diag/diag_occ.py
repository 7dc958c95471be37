"""Forced-occupancy diagnostic (
profiles/r02/diag_forced_occupancy.jsonl). NOT a product path: it needs a
diagnostic build of libcrsd.so in which launch_fn (csrc/jit.cpp) pads the
dynamic shared memory so that at most CRSD_DIAG_OCC CTAs fit per SM:

    if (const char *e = getenv("CRSD_DIAG_OCC")) {
        const int occ = atoi(e);
        if (occ > 0) {
            const unsigned want = (unsigned)((228 * 1024) / occ - 1280 - 128) / 128 * 128;
            if (want > smem) smem = want;
            driver().set_attr(fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)smem);
        }
    }

With the product build the variable has no effect. (The per-launch
cuFuncSetAttribute of the diagnostic build costs a little on its own: compare
forced values with each other, not with "0".)

usage: python scripts/diag/diag_occ.py c3:f64:one c3:f64 c2:f64
"""
import json, os, sys
import torch
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import bench
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix
PEAK = bench.measured_peaks()[0]
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
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, variant=4, tune=0x2 if "one" in case else 0)
    ub = A.info()["unique_bytes_beta0"]
    for rep in range(3):
        for occ in ["0", "4", "3", "2", "1"]:
            os.environ["CRSD_DIAG_OCC"] = occ
            ms = t(A, x, y)
            print(json.dumps({"case": case, "occ": occ, "rep": rep, "ms": round(ms, 5), "frac": round(ub / (ms * 1e-3) / 1e9 / PEAK, 4), "launches": A.last_launch_count()}), flush=True)
