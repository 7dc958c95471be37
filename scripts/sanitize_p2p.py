#!/usr/bin/env python
"""Two real ranks on cuda:0 through the peer-memory transport (halo exchange,
allreduce, distributed CG), for compute-sanitizer with --target-processes all.
Reuses the GPU test's worker (tests/test_gpu_p2p.py) and checks its parity.

usage: compute-sanitizer --target-processes all --tool memcheck python scripts/sanitize_p2p.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CRSD_P2P_TIMEOUT_S", "120")  # sanitized kernels are slow

from tests import test_gpu_p2p as t  # noqa: E402


def main():
    bad = 0
    for case, world, variant, mode in (("c3", 2, 0, "mailbox"), ("multihop", 3, 4, "mailbox"), ("c3", 2, 0, "direct"),
                                       ("multihop", 4, 0, "direct"), ("cg7pt", 2, 0, "direct")):
        res = t._run(case, world, variant, mode=mode)
        for r in res:
            if "errs" in r:
                ok = max(r["errs"]) <= 1e-12
            else:
                ok = r["rr_rel"] <= 1e-11 and r["x_rel"] <= 1e-12
            bad += not ok
            print(f"{case} {mode} world {world} rank {r['rank']}: {'ok' if ok else 'FAIL'}", flush=True)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
