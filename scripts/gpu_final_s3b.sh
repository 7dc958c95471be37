#!/bin/bash
# Closing evidence after the concurrent-range change: sanitizers on the forced
# range split, bench lines (default, C2 f32, C3 f64/f32, C4 f32), smoke.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/final2
mkdir -p $O
timeout 300 python __graft_entry__.py --smoke > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
for tl in memcheck racecheck; do
  timeout 900 compute-sanitizer --tool $tl --error-exitcode 9 python scripts/sanitize.py > $O/sanitize_$tl.log 2>&1; echo "rc=$?" >> $O/sanitize_$tl.log
done
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
for cfg in "c2 f32 512" "c3 f64 256" "c3 f32 256" "c4 f32 512"; do
  set -- $cfg
  timeout 900 python bench.py --no-cpu --config $1 --dtype $2 --mrows $3 > $O/bench_$1_$2.json 2> $O/bench_$1_$2.err
done
timeout 1200 ncu --set full --clock-control none -k regex:crsd_jit -s 15 -c 5 -o $O/prof_c3_f64_step -f python bench.py --config c3 --dtype f64 --steps 2 --warmup 3 --no-cpu > $O/ncu_c3.log 2>&1
python scripts/ncu_summary.py $O/prof_c3_f64_step.ncu-rep --bytes 1357444604 > $O/ncu_c3_f64_step.json 2>&1
echo done
