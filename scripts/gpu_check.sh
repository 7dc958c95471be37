#!/bin/bash
# One gpurun pass: smoke, GPU tests, bench lines, ncu launch list + full captures.
# Env: SKIP_TESTS=1, BENCH_SET="c2:f64:tma c3:f64:ldg ...", NCU_SET="c2:f64:tma ..."
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvsmi.txt 2>&1
for o in "2" "1 2" "3" "1 3"; do timeout 120 python scripts/debug_first_launch.py $o >> gpurun_out/debug_first_launch.log 2>&1; done
if [ -z "$SKIP_TESTS" ]; then
  timeout 300 python __graft_entry__.py --smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
  timeout 1800 python -m pytest tests -m gpu -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
fi
for cfg in ${BENCH_SET:-c2:f64:ldg c2:f64:tma c2:f64:pipe c2:f32:tma c2:f32:pipe c3:f64:ldg c3:f64:tma c3:f64:pipe c3:f32:ldg c3:f32:pipe}; do
  IFS=: read c d v m <<< "$cfg"
  mr=""; [ -n "$m" ] && mr="--mrows $m"
  timeout 600 python bench.py --no-cpu --config $c --dtype $d --variant $v $mr ${BENCH_ARGS} > gpurun_out/bench_${c}_${d}_${v}${m}.json 2> gpurun_out/bench_${c}_${d}_${v}${m}.err
done
for cfg in ${NCU_SET:-c2:f64:pipe c3:f64:pipe}; do
  IFS=: read c d v <<< "$cfg"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_spmv -s 5 -c 1 -o gpurun_out/prof_${c}_${d}_${v} -f python bench.py --steps 10 --warmup 5 --no-cpu --config $c --dtype $d --variant $v > gpurun_out/ncu_${c}_${d}_${v}.log 2>&1
done
echo done
