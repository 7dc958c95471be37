#!/usr/bin/env python
"""Probe: can two NCCL ranks share one GPU (both on cuda:0)? Diagnostic only.

torchrun --nproc-per-node 2 --master-addr 127.0.0.1 scripts/nccl_shared_gpu_probe.py
Tries torch.distributed NCCL (all_reduce, send/recv) and libcrsd's own
communicator (crsd_comm_init_rank) with every rank on device 0.
"""
import os
import sys

import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    dist.init_process_group("gloo", init_method="env://")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(0)
    out = {}
    try:
        from paper_conf_icpp_sunzwzyr11_b200 import Comm

        c = Comm(rank, world, 0)
        out["crsd_comm"] = "ok"
        c.close()
    except Exception as e:  # noqa: BLE001
        out["crsd_comm"] = f"fail: {e}"[:300]
    print(rank, out, flush=True)


if __name__ == "__main__":
    main()
