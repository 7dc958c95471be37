#!/bin/bash
# Round 2: e2e timelines (C2 / C5), C3 mrows sweep, C3 vs C3ns source-level ncu.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02e
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for ch in 0 8 16 32; do timeout 600 python scripts/e2e_trace.py c2 $ch > $O/e2e_c2_$ch.jsonl 2> $O/e2e_c2_$ch.err; done
timeout 900 python scripts/e2e_trace.py c5 0 > $O/e2e_c5.jsonl 2> $O/e2e_c5.err
SWEEP_SET="win=0,0" SWEEP_REPS=3 timeout 900 python scripts/sweep.py c3:f64:128 c3:f64:256 c3ns:f64:256 c3:f32:128 > $O/sweep_mrows.jsonl 2> $O/sweep_mrows.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 27 -c 1 -o $O/prof_c3_f64_big -f python bench.py --config c3 --steps 10 --warmup 5 --no-cpu > $O/ncu_c3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 27 -c 1 -o $O/prof_c3ns_f64_big -f python bench.py --config c3ns --steps 10 --warmup 5 --no-cpu > $O/ncu_c3ns.log 2>&1
echo done
