#!/bin/bash
# Evidence run: smoke, GPU tests, default bench (+cpu baseline), reference arm,
# AUTO bench lines, ncu launch list of the default bench, ncu full captures of
# the AUTO kernel per workload, CG throughput, compute-sanitizer. Everything
# lands in gpurun_out/ (summaries are copied to profiles/).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvsmi.txt 2>&1
timeout 300 python __graft_entry__.py --smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
for cfg in "c2 f32" "c3 f64" "c3 f32" "c4 f32"; do
  set -- $cfg
  timeout 900 python bench.py --no-cpu --config $1 --dtype $2 > gpurun_out/bench_$1_$2.json 2> gpurun_out/bench_$1_$2.err
done
timeout 900 python bench.py --no-cpu --config c3 --dtype f32 --mrows 256 > gpurun_out/bench_c3_f32_m256.json 2> gpurun_out/bench_c3_f32_m256.err
for d in f64 f32; do timeout 600 python bench.py --workload cg --dtype $d > gpurun_out/bench_cg_$d.json 2> gpurun_out/bench_cg_$d.err; done
timeout 600 ncu --set full --clock-control none -k regex:cg_ -s 12 -c 3 -o gpurun_out/prof_cg_f64 -f python bench.py --workload cg --steps 20 --warmup 3 > gpurun_out/ncu_cg.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_default.csv python bench.py --steps 20 --warmup 3 --no-cpu > /dev/null 2>&1
for cfg in "c2 f64" "c2 f32" "c3 f64" "c3 f32" "c4 f32"; do
  set -- $cfg
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_ -s 5 -c 1 -o gpurun_out/prof_$1_$2_auto -f python bench.py --steps 10 --warmup 5 --no-cpu --config $1 --dtype $2 > gpurun_out/ncu_$1_$2.log 2>&1
done
for t in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $t --error-exitcode 9 python scripts/sanitize.py > gpurun_out/sanitize_$t.log 2>&1; echo "rc=$?" >> gpurun_out/sanitize_$t.log
done
echo done
