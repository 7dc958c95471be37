#!/bin/bash
# Quick verification pass: GPU tests, CG throughput (fused / unfused (p,q)),
# racecheck of the JIT + CG paths, optional JIT mrows sweep. Output in gpurun_out/.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 300 python __graft_entry__.py --smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
( for d in f64 f32; do timeout 300 python scripts/cg_bench.py 256 2000 $d; CRSD_CG_FUSED_DOT=1 timeout 300 python scripts/cg_bench.py 256 2000 $d; done ) > gpurun_out/cg_bench.jsonl 2>&1
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/sanitize.py > gpurun_out/sanitize_racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/sanitize_racecheck.log
if [ -n "$SWEEP_CASES" ]; then SWEEP_VARIANTS=${SWEEP_VARIANTS:-jit} timeout 1200 python scripts/sweep.py $SWEEP_CASES > gpurun_out/sweep.jsonl 2>&1; fi
echo done
