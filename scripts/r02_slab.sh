#!/bin/bash
# Round 2 (session 2): scatter slab A/B (CRSD_TUNE_JIT_NO_SLAB) + parity.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02s2
mkdir -p $O
nvidia-smi > $O/nvsmi3.txt 2>&1
timeout 1800 python -m pytest tests/test_gpu_spmv.py tests/test_gpu_p2p.py -m gpu -q -x -k "staging_chunks or random_diagonal or c1 or c3 or pdl or dense or p2p or dist" > $O/pytest_slab.log 2>&1; echo "pytest rc=$?" >> $O/pytest_slab.log
SWEEP_SET="def=0,0;noslab=0,0x100" SWEEP_REPS=4 timeout 1500 python scripts/sweep.py c3:f64 c3:f32 > $O/sweep_slab.jsonl 2> $O/sweep_slab.err
echo done
