#!/bin/bash
# Round 2 closing evidence after the PDL / scatter-slab codelets: build, smoke,
# full GPU suite, the driver's bench command, the reference arm, the ncu launch
# list of the default command, ncu --set full captures (C5, C3 f64,
# C3 f32). No compute-sanitizer (closed on this pool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02s2final2
mkdir -p $O
nvidia-smi > $O/nvsmi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python __graft_entry__.py --smoke > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 3000 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 900 python bench.py --steps 100 --warmup 10 > $O/bench100.json 2> $O/bench100.err
timeout 900 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > $O/ref.json 2> $O/ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 500 --csv --log-file $O/launches_default.csv python bench.py --steps 5 --warmup 3 --no-cpu > $O/launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 3 -c 1 -o $O/prof_c5_f64 -f python bench.py --steps 5 --warmup 3 --no-cpu --no-sub > $O/ncu_c5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 5 -c 1 -o $O/prof_c3_f64 -f python bench.py --config c3 --steps 10 --warmup 5 --no-cpu > $O/ncu_c3_f64.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 5 -c 1 -o $O/prof_c3_f32 -f python bench.py --config c3 --dtype f32 --steps 10 --warmup 5 --no-cpu > $O/ncu_c3_f32.log 2>&1
echo done
