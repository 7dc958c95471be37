#!/bin/bash
# mrows 192 (4 CTAs/SM for C3 f64) vs 256; f32 384 vs 256.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02s4; mkdir -p $O
for r in 1 2; do
  SWEEP_SET="win=0,0" SWEEP_REPS=1 timeout 900 python scripts/sweep.py c3:f64:192 c3:f64:256 c3:f32:384 c3:f32:256 c2:f64:192 c2:f64:256 > $O/sweep_$r.jsonl 2>> $O/err.txt
done
echo done
