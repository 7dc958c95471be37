#!/bin/bash
# Session-3 evidence run: smoke, every GPU test, bench lines (default, reference
# arm, C2 f32, C3, C4 occupancy ranges), ncu launch list of the default bench,
# ncu full captures of the default kernel and of one whole C4 step (6 launches).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/final
O=gpurun_out/final
nvidia-smi > $O/nvsmi.txt 2>&1
timeout 300 python __graft_entry__.py --smoke > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $O/bench_reference.json 2> $O/bench_reference.err
for cfg in "c2 f32 512" "c3 f64 256" "c3 f32 256" "c4 f32 512"; do
  set -- $cfg
  timeout 900 python bench.py --no-cpu --config $1 --dtype $2 --mrows $3 > $O/bench_$1_$2.json 2> $O/bench_$1_$2.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $O/launches_default.csv python bench.py --steps 20 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 5 -c 1 -o $O/prof_c2_f64 -f python bench.py --steps 5 --warmup 5 --no-cpu > $O/ncu_c2.log 2>&1
timeout 1200 ncu --set full --clock-control none -k regex:crsd_jit -s 18 -c 6 -o $O/prof_c4_f32_step -f python bench.py --config c4 --dtype f32 --mrows 512 --steps 2 --warmup 3 --no-cpu > $O/ncu_c4.log 2>&1
python scripts/ncu_summary.py $O/prof_c2_f64.ncu-rep --bytes 1205862400 > $O/ncu_c2_f64.json 2>&1
python scripts/ncu_summary.py $O/prof_c4_f32_step.ncu-rep --bytes 5543477248 > $O/ncu_c4_f32_step.json 2>&1
echo done
