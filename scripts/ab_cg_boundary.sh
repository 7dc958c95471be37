#!/bin/bash
# CG under MPS (2 ranks on cuda:0): boundary placement x graph batches.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/ab_cg
for g in 0 1; do for b in 0 1; do
  CRSD_CG_NO_GRAPH=$g CRSD_CG_BOUNDARY=$b MPS_NS="2" MPS_ARGS="--workload cg --steps 500" bash scripts/mps_share_bench.sh
  mv gpurun_out/bench_mps2.json gpurun_out/ab_cg/cg_nograph${g}_boundary${b}.json
done; done
for f in gpurun_out/ab_cg/*.json; do python -c "
import json; j=json.load(open('$f')); print('$f'.split('/')[-1], j['value'], j['ms_per_step'])"; done
