#!/bin/bash
# Round 2: fused halo receive on the GPU (p2p tests), sanitizers on it, MPS overlap trace, bench.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02g
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_cg.py -m gpu -q -x > $O/pytest_p2p.log 2>&1; echo "rc=$?" >> $O/pytest_p2p.log
timeout 1500 compute-sanitizer --tool memcheck --target-processes all --print-limit 20 python scripts/sanitize_p2p.py > $O/san_p2p_memcheck.txt 2>&1; echo "rc=$?" >> $O/san_p2p_memcheck.txt
timeout 1500 compute-sanitizer --tool racecheck --target-processes all --print-limit 20 python scripts/sanitize_p2p.py > $O/san_p2p_racecheck.txt 2>&1; echo "rc=$?" >> $O/san_p2p_racecheck.txt
OV_CFGS="c2:2:direct c5:2:direct c2:4:direct" bash scripts/r02_overlap.sh > $O/overlap.log 2>&1
timeout 900 python bench.py --steps 100 --warmup 10 > $O/bench.json 2> $O/bench.err
echo done
