#!/bin/bash
# Round 2 closing evidence: build, smoke, full GPU suite, initcheck, default bench (driver command),
# reference arm, ncu launch list of the default command.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02final
mkdir -p $O
nvidia-smi > $O/nvsmi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python __graft_entry__.py --smoke > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 3600 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 1200 compute-sanitizer --tool initcheck --print-limit 20 python scripts/sanitize.py > $O/san_initcheck.txt 2>&1; echo "rc=$?" >> $O/san_initcheck.txt
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 900 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > $O/ref.json 2> $O/ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 500 --csv --log-file $O/launches_default.csv python bench.py --steps 5 --warmup 3 --no-cpu > $O/launches.log 2>&1
echo done
