#!/usr/bin/env python
"""SASS instruction histogram of the JIT codelets the bench runs (no GPU needed:
crsd_jit_cubin compiles the generated source with NVRTC for sm_100a; cuobjdump
disassembles it). Evidence that the data path is Blackwell bulk copies
(UBLKCP) completing on mbarriers (SYNCS.*), that the FMAs read shared memory
(LDS), and that no per-nonzero index is loaded: the only global loads (LDG)
are the scatter records / scatter x gathers and the guarded edge path.

usage: python scripts/sass_histogram.py > profiles/r02/sass_histogram.json
"""
import collections
import json
import os
import re
import subprocess
import sys
import tempfile

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import gen  # noqa: E402
from gen import fast  # noqa: E402
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix  # noqa: E402

CUOBJDUMP = "/usr/local/cuda/bin/cuobjdump"


def cases():
    a = gen.config3()
    yield "C3 f64 (full size)", CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val, host_only=True)
    yield "C3 f32 (full size)", CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val.astype(np.float32), host_only=True)
    del a
    d = (256, 256, 256)
    p, c, v = fast.stencil(d, bench._stencil_disps("7pt", d), False, True, 2, None, 0, 256**3, csr=True)
    yield "C2 f64 (full size)", CRSDMatrix.from_csr(256**3, 256**3, p, c, v, host_only=True)
    d = (768, 768, 768)
    n = 768**3
    N, rb, re = bench.rank_rows("c5", 8, 0)
    p, c, v = fast.stencil(d, bench._stencil_disps("7pt", d), False, False, 5, None, rb, re, csr=True)
    yield "C5 f64 (rows of rank 0 of 8: the same 9 codelets as the one-GPU handle; a smaller lookup tree)", \
        CRSDMatrix.from_csr(n, n, p, c, v, host_only=True, row_range=(rb, re))
    n4 = 100_000_000
    p, c, v = fast.band(n4, gen.matrices.c4_ranges(n4), 4, 0, n4, csr=True)
    yield "C4 f32 (full size)", CRSDMatrix.from_csr(n4, n4, p, c, v.astype(np.float32), host_only=True)


def histogram(cubin: bytes):
    with tempfile.NamedTemporaryFile(suffix=".cubin") as f:
        f.write(cubin)
        f.flush()
        sass = subprocess.run([CUOBJDUMP, "-sass", f.name], capture_output=True, text=True, check=True).stdout
    ops = collections.Counter()
    for line in sass.splitlines():
        m = re.match(r"\s*/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", line)
        if m:
            ops[m.group(1)] += 1
    fam = collections.Counter()
    for op, k in ops.items():
        fam[op.split(".")[0]] += k
    return ops, fam


def main():
    out = {"how": "crsd_jit_cubin (NVRTC, sm_100a) | cuobjdump -sass; static instruction counts of the whole module "
                  "(crsd_jit, crsd_jit_halo, and crsd_jit_rs where register staging is used: C3 f64). The launch plan "
                  "is the one a device handle makes (148 SMs): one-launch handles carry programmatic dependent launch "
                  "(PREEXIT = griddepcontrol.launch_dependents, ACQBULK = griddepcontrol.wait); C4 (occupancy-class "
                  "ranges) and the row-partitioned C5 rank block do not",
           "kernels": []}
    for name, A in cases():
        inf = A.info()
        ops, fam = histogram(A.jit_cubin())
        rec = {
            "workload": name,
            "dtype": "f64" if inf["dtype"] == 1 else "f32",
            "mrows": inf["mrows"],
            "patterns": inf["npat"],
            "instances": inf["ninst"],
            "families": {k: fam[k] for k in ("UBLKCP", "SYNCS", "LDS", "LDG", "DFMA", "FFMA", "STG", "BAR", "SHFL", "PREEXIT", "ACQBULK")},
            "total_instructions": sum(ops.values()),
            "ldg_variants": {k: v for k, v in sorted(ops.items()) if k.startswith("LDG")},
            "syncs_variants": {k: v for k, v in sorted(ops.items()) if k.startswith("SYNCS")},
        }
        out["kernels"].append(rec)
        print(name, rec["families"], file=sys.stderr, flush=True)
        A.close()
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
