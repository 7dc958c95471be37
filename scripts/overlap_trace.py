#!/usr/bin/env python
"""Overlap evidence for crsd_spmv_dist: a CUPTI kernel trace
(torch.profiler / Kineto, which records every kernel of the process,
including the driver-API launches of the JIT codelets) of K row-partitioned
SpMV steps, and per step the share of the halo path (exchange kernels +
boundary segments, on the comm stream) that runs inside the span of the
interior segments (on the compute stream).

Run under torchrun with every rank on cuda:0 and CUDA MPS active (the
gpurun boxes have one GPU; under MPS the ranks' kernels run concurrently):
    torchrun --nproc-per-node 2 scripts/overlap_trace.py [c2|c5] [direct|mailbox]
Writes gpurun_out/overlap/trace_rank<r>.json (chrome trace) and prints one
JSON summary line per rank.
"""
import json
import os
import re
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
    mode = sys.argv[2] if len(sys.argv) > 2 else "direct"
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(0)
    from paper_conf_icpp_sunzwzyr11_b200 import P2PComm

    A, desc, (rb, rend), N, _ = bench.build(cfg, "f64", world, rank, 0, nthreads=max(1, bench.host_cores() // world))
    lo, nloc, hi = A.x_layout()
    comm = P2PComm(rank, world, 0, mailbox_bytes=max(1 << 20, 4 * (lo + hi) * 8))
    A.dist_bind(comm)
    if mode == "direct":
        xp = A.dist_x_alloc(comm)
    else:
        xp = torch.zeros(lo + nloc + hi, dtype=torch.float64, device="cuda:0")
    xp[lo : lo + nloc] = torch.from_numpy(np.random.default_rng(rank).uniform(-1, 1, nloc)).to("cuda:0")
    y = torch.empty(nloc, dtype=torch.float64, device="cuda:0")
    for _ in range(10):
        A.spmv_dist(xp, y, 1.0, 0.0, comm)
    torch.cuda.synchronize()
    dist.barrier()
    K = 8
    from torch.profiler import ProfilerActivity, profile

    with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
        for _ in range(K):
            A.spmv_dist(xp, y, 1.0, 0.0, comm)
        torch.cuda.synchronize()
    dist.barrier()
    assert comm.error() == 0
    out_dir = os.path.join(ROOT, "gpurun_out", "overlap")
    os.makedirs(out_dir, exist_ok=True)
    path = os.path.join(out_dir, f"trace_{cfg}_{mode}_rank{rank}.json")
    prof.export_chrome_trace(path)
    # kernels of this process: name, stream, start, end (us)
    with open(path) as f:
        tr = json.load(f)
    ks = [e for e in tr["traceEvents"] if e.get("cat") == "kernel"]
    ks.sort(key=lambda e: e["ts"])
    streams = sorted({e["args"].get("stream") for e in ks})
    # the comm stream carries the p2p_* kernels and the boundary segments;
    # the compute stream the interior segments (one crsd_jit launch per call
    # for these matrices). A call = one interior launch and the comm-stream
    # kernels that follow it up to the next interior launch.
    comm_stream = next(e["args"]["stream"] for e in ks if "p2p" in e["name"])
    inter = [e for e in ks if e["args"].get("stream") != comm_stream]
    comm_k = [e for e in ks if e["args"].get("stream") == comm_stream]
    recs = []
    for i, e in enumerate(inter):
        i0, i1 = e["ts"], e["ts"] + e["dur"]
        nxt = inter[i + 1]["ts"] if i + 1 < len(inter) else float("inf")
        mine = [c for c in comm_k if i0 <= c["ts"] < nxt]
        if not mine:
            continue
        tl = [(re.search(r"p2p_\w+", c["name"]).group(0) if "p2p" in c["name"] else "boundary " + c["name"],
               round(c["ts"] - i0, 1), round(c["ts"] + c["dur"] - i0, 1)) for c in mine]
        busy = sum(c["dur"] for c in mine)
        inside = sum(max(0.0, min(c["ts"] + c["dur"], i1) - max(c["ts"], i0)) for c in mine)
        recs.append({"interior_us": round(i1 - i0, 1), "comm_path_end_us": round(max(c["ts"] + c["dur"] for c in mine) - i0, 1),
                     "comm_kernel_us_inside_interior": round(inside, 1), "comm_kernel_us": round(busy, 1),
                     "timeline_us_from_interior_start": tl})
    print(json.dumps({"rank": rank, "world": world, "config": desc, "mode": mode, "streams": len(streams),
                      "calls": recs}), flush=True)
    comm.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
