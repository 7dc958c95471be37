#!/bin/bash
# The SCALE command path (default config C5, self-launched ranks, peer-memory one-sided puts)
# with N ranks sharing cuda:0 under CUDA MPS: functional check of the 2/4/8-rank C5 flow.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02s8; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
(free -g) > $O/mem.txt
MPS=$(command -v nvidia-cuda-mps-control)
export CUDA_MPS_PIPE_DIRECTORY=/tmp/crsd_mps_pipe CUDA_MPS_LOG_DIRECTORY=/tmp/crsd_mps_log
mkdir -p $CUDA_MPS_PIPE_DIRECTORY $CUDA_MPS_LOG_DIRECTORY
$MPS -d > $O/mps.log 2>&1
sleep 2
for n in 2 4 8; do
  timeout 1500 python bench.py --gpus $n --share-gpu --transport p2p --steps 20 --warmup 5 > $O/bench_c5_share$n.json 2> $O/bench_c5_share$n.err
  echo "n=$n rc=$?" >> $O/mps.log
done
echo quit | $MPS >> $O/mps.log 2>&1
echo done
