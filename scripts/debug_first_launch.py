"""Fresh-process check: does the first kernel launched in a process matter?"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gen
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix
order = sys.argv[1:]
torch.cuda.set_device(0)
a = gen.config1()
for v in order:
    A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, device=0, variant=int(v))
    x = torch.rand(a.ncols, dtype=torch.float64, device="cuda:0")
    y = torch.zeros(a.nrows, dtype=torch.float64, device="cuda:0")
    try:
        A.spmv(x, y, 1.0, 0.0); torch.cuda.synchronize(); print("variant", v, "ok", A.info()["smem_bytes"])
    except Exception as e:
        print("variant", v, "FAIL", e)
