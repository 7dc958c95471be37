#!/bin/bash
# CG throughput with the round-2 codelets, and the default bench with the C4 record.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02cg
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for d in f64 f32; do timeout 600 python bench.py --workload cg --dtype $d --steps 2000 --warmup 300 > $O/cg_$d.json 2> $O/cg_$d.err; done
timeout 1200 python bench.py --steps 50 --warmup 5 > $O/bench.json 2> $O/bench.err
echo done
