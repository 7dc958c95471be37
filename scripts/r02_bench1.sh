#!/bin/bash
# Round 2: first run of the restructured bench (C5 default + C3 f64/f32 sub-records), reference arm.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02b1
mkdir -p $O
(free -g; nproc; lscpu | head -20) > $O/host.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python bench.py --steps 50 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > $O/ref.json 2> $O/ref.err
timeout 600 python bench.py --gpus 2 --share-gpu --transport p2p --config c2 --steps 20 --warmup 3 > $O/share2.json 2> $O/share2.err
echo done
