#!/bin/bash
# A/B runs of this session: (1) JIT scatter head records on C3 (CRSD_JIT_SCAT_HEAD
# 0/1, interleaved); (2) dist exchange order/grid under MPS (N ranks on cuda:0).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for rep in 1 2; do
  for h in 0 1; do
    CRSD_JIT_SCAT_HEAD=$h SWEEP_VARIANTS=jit timeout 600 python scripts/sweep.py c3:f64 c3:f32:256 c3:f32:512 2>&1 | sed "s/^/head=$h rep=$rep /" >> gpurun_out/ab_scat_head.jsonl
  done
done
export MPS_NS="1 2 4"
MPS_ARGS="" bash scripts/mps_share_bench.sh; mkdir -p gpurun_out/mps_new; mv gpurun_out/bench_mps* gpurun_out/mps.log gpurun_out/mps_new/
CRSD_DIST_EXCHANGE_FIRST=1 CRSD_P2P_GRID=32 MPS_NS="2 4" bash scripts/mps_share_bench.sh; mkdir -p gpurun_out/mps_old; mv gpurun_out/bench_mps* gpurun_out/mps.log gpurun_out/mps_old/
echo done
