#!/bin/bash
# Round 2: sanitizers on the new codelets and the direct-put transport, overlap traces under MPS, small sweep.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02san
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize.py > $O/san_$tool.txt 2>&1; echo "rc=$?" >> $O/san_$tool.txt
done
timeout 1500 compute-sanitizer --tool memcheck --target-processes all --print-limit 20 python scripts/sanitize_p2p.py > $O/san_p2p_memcheck.txt 2>&1; echo "rc=$?" >> $O/san_p2p_memcheck.txt
OV_CFGS="c2:2:direct c2:2:mailbox c5:2:direct c2:4:direct" bash scripts/r02_overlap.sh > $O/overlap.log 2>&1
SWEEP_SET="win256=0,0" SWEEP_REPS=3 timeout 900 python scripts/sweep.py c3:f64:128 c3:f64:256 c3:f32:128 > $O/sweep_mrows.jsonl 2> $O/sweep_mrows.err
timeout 600 python scripts/e2e_probe.py 8 16 32 > $O/e2e_c2_chunks.txt 2>&1
echo done
