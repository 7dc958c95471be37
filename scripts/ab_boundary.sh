#!/bin/bash
# A/B of the boundary placement under MPS (ranks share cuda:0): boundary
# segments on the comm stream concurrent with the interior (default) vs
# serial after the interior (CRSD_DIST_BOUNDARY_SERIAL=1); SpMV and CG.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/ab_boundary
for rep in 1 2; do
  for ser in 0 1; do
    CRSD_DIST_BOUNDARY_SERIAL=$ser MPS_NS="2 4" bash scripts/mps_share_bench.sh
    for n in 2 4; do mv gpurun_out/bench_mps$n.json gpurun_out/ab_boundary/spmv_ser${ser}_n${n}_rep$rep.json; done
  done
done
for ser in 0 1; do
  CRSD_DIST_BOUNDARY_SERIAL=$ser MPS_NS="2 4" MPS_ARGS="--workload cg --steps 500" bash scripts/mps_share_bench.sh
  for n in 2 4; do mv gpurun_out/bench_mps$n.json gpurun_out/ab_boundary/cg_ser${ser}_n${n}.json; done
done
for f in gpurun_out/ab_boundary/*.json; do python -c "
import json,sys; j=json.load(open('$f')); print('$f'.split('/')[-1], j['value'], j['ms_per_step'])"; done
