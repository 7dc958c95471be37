#!/bin/bash
# Round 2 (session 2): PDL as the default for one-launch handles.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02s2
mkdir -p $O
nvidia-smi > $O/nvsmi2.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_spmv.py tests/test_gpu_cg.py tests/test_gpu_bench.py -m gpu -q > $O/pytest_pdl2.log 2>&1; echo "pytest rc=$?" >> $O/pytest_pdl2.log
SWEEP_SET="def=0,0;nopdl=0,0x80" SWEEP_REPS=3 timeout 1500 python scripts/sweep.py c3:f32 c2:f64 c2:f32 c3:f64 > $O/sweep_pdl2.jsonl 2> $O/sweep_pdl2.err
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $O/bench_pdl.json 2> $O/bench_pdl.err
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_spmv.py -m gpu -q -k "pdl_dependent_chain and (c2 or c3)" > $O/san_memcheck_pdl.txt 2>&1; echo "rc=$?" >> $O/san_memcheck_pdl.txt
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python -m pytest tests/test_gpu_spmv.py -m gpu -q -k "pdl_dependent_chain and c3" > $O/san_racecheck_pdl.txt 2>&1; echo "rc=$?" >> $O/san_racecheck_pdl.txt
echo done
