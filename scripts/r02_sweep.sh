#!/bin/bash
# Round 2: JIT staging-chunk / issue A/B (parity subset first, then the sweep).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/r02
O=gpurun_out/r02
nvidia-smi > $O/nvsmi.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_spmv.py -m gpu -q -x -k "jit or c1_parity or c3_reduced or c2_reduced or c4_reduced or occupancy" > $O/pytest_jit.log 2>&1; echo "pytest rc=$?" >> $O/pytest_jit.log
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.sw_power_cap --format=csv -lms 500 > $O/clocks.csv &
SMI=$!
SWEEP_SET="${SWEEP_SET:-one=-1,0;win=0,0;k4=4,0;k2=2,0;desc=0,1;onedesc=-1,1}" SWEEP_REPS=${SWEEP_REPS:-3} timeout 1500 python scripts/sweep.py ${SWEEP_CASES:-c3:f64 c3:f32:256 c3:f32:512 c2:f64 c2:f32} > $O/sweep.jsonl 2> $O/sweep.err
kill $SMI
echo done
