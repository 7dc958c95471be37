#!/bin/bash
# Round 2: full GPU suite + smoke + default bench + reference arm + ncu captures.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02f
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python __graft_entry__.py --smoke > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 3000 python -m pytest tests -m gpu -q ${PYTEST_ARGS} > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 900 python bench.py --steps 100 --warmup 10 > $O/bench.json 2> $O/bench.err
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > $O/ref.json 2> $O/ref.err
# launch list of the default bench command (cold, serialised: compare shares)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_default.csv python bench.py --steps 5 --warmup 3 --no-cpu > $O/launches_default.log 2>&1
# full captures: C5 (one launch), C3 f64 (one whole step = 5 range launches), C3 f32
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 3 -c 1 -o $O/prof_c5_f64 -f python bench.py --steps 5 --warmup 3 --no-cpu --no-sub > $O/ncu_c5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 25 -c 5 -o $O/prof_c3_f64 -f python bench.py --config c3 --steps 10 --warmup 5 --no-cpu > $O/ncu_c3_f64.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 5 -c 1 -o $O/prof_c3_f32 -f python bench.py --config c3 --dtype f32 --steps 10 --warmup 5 --no-cpu > $O/ncu_c3_f32.log 2>&1
echo done
