#!/bin/bash
# Round 2 (session 2): register staging as the default where it yields one launch.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02s2
mkdir -p $O
timeout 2400 python -m pytest tests/test_gpu_spmv.py tests/test_gpu_cg.py -m gpu -q > $O/pytest_rs2.log 2>&1; echo "pytest rc=$?" >> $O/pytest_rs2.log
echo done
