#!/bin/bash
# Round 2 sweep 2: scatter cost on the new codelets, C4, and one ncu capture of C3 f64.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02s2
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.sw_power_cap --format=csv -lms 500 > $O/clocks.csv &
SMI=$!
SWEEP_SET="win=0,0;one=-1,0;desc=0,1;k9=9,0;k3=3,0" SWEEP_REPS=3 timeout 1500 python scripts/sweep.py c3:f64 c3ns:f64 c3:f32:256 c3ns:f32:256 c4:f32:512 > $O/sweep.jsonl 2> $O/sweep.err
kill $SMI
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 5 -c 1 -o $O/prof_c3_f64 -f python bench.py --steps 10 --warmup 5 --no-cpu --config c3 --dtype f64 > $O/ncu_c3_f64.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:crsd_jit -s 5 -c 1 -o $O/prof_c3_f32 -f python bench.py --steps 10 --warmup 5 --no-cpu --config c3 --dtype f32 --mrows 256 > $O/ncu_c3_f32.log 2>&1
echo done
