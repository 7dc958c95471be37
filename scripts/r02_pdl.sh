#!/bin/bash
# Round 2 (session 2): programmatic dependent launch A/B (CRSD_TUNE_JIT_PDL).
# Parity subset first (PDL chain, chunk/issue settings, occupancy ranges), then
# the interleaved sweep: default vs PDL, plus PDL with one launch.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02s2
mkdir -p $O
nvidia-smi > $O/nvsmi.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_spmv.py -m gpu -q -x -k "pdl or staging_chunks or occupancy" > $O/pytest_pdl.log 2>&1; echo "pytest rc=$?" >> $O/pytest_pdl.log
SWEEP_SET="${SWEEP_SET:-def=0,0;pdl=0,0x80;pdl1=0,0x82;seq=0,0x8}" SWEEP_REPS=${SWEEP_REPS:-3} timeout 1500 python scripts/sweep.py ${SWEEP_CASES:-c3:f64 c3:f32 c2:f64 c4:f32:512} > $O/sweep_pdl.jsonl 2> $O/sweep_pdl.err
echo done
