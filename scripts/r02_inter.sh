#!/bin/bash
# Round 2 (session 2): interleaved single launch A/B (CRSD_TUNE_JIT_INTERLEAVE) + parity.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02s2
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_spmv.py -m gpu -q -x -k "interleave" > $O/pytest_inter.log 2>&1; echo "pytest rc=$?" >> $O/pytest_inter.log
SWEEP_SET="def=0,0;inter=0,0x200" SWEEP_REPS=4 timeout 1500 python scripts/sweep.py c3:f64 c4:f32:512 > $O/sweep_inter.jsonl 2> $O/sweep_inter.err
echo done
