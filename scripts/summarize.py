#!/usr/bin/env python
"""Markdown tables from the committed evidence in profiles/ (bench lines,
sweeps, ncu summaries) for DESIGN.md §12."""
import glob
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
P = os.path.join(ROOT, "profiles")


def bench_table(pattern):
    rows = []
    for f in sorted(glob.glob(os.path.join(P, pattern))):
        try:
            j = json.load(open(f))
        except Exception:
            continue
        if "roofline" not in j:
            continue
        r = j["roofline"]
        e = j.get("e2e") or {}
        rows.append(
            f"| {os.path.basename(f)} | {j['config']['workload'][:60]} | {j['dtype']} | {r['kernel']} | {j['value']:.0f} | {r['achieved']:.0f} | {r['frac']:.3f} | {r.get('copy_gbs_this_box', '')} | {e.get('value', '')} | {e.get('ms_per_step', '')} | {e.get('transfer_bound_ms', '')} |"
        )
    hdr = "| file | workload | dtype | kernel | GFLOP/s | GB/s (algorithmic) | frac of 6,550 | box copy GB/s | e2e GFLOP/s | e2e ms | transfer bound ms |\n|---|---|---|---|---|---|---|---|---|---|---|"
    return hdr + "\n" + "\n".join(rows)


def sweep_table(fname):
    rows = []
    for line in open(os.path.join(P, fname)):
        j = json.loads(line)
        if "frac" not in j:
            continue
        rows.append(f"| {j['case']} | {j.get('mrows', '')} | {j['variant']} | {j.get('shape')} | {j['ms']} | {j['GBps']} | {j['frac']} |")
    return "| case | mrows | variant | shape | ms | GB/s | frac |\n|---|---|---|---|---|---|---|\n" + "\n".join(rows)


if __name__ == "__main__":
    what = sys.argv[1] if len(sys.argv) > 1 else "bench"
    if what == "bench":
        print(bench_table(sys.argv[2] if len(sys.argv) > 2 else "r01_bench_*.json"))
    else:
        print(sweep_table(what))
