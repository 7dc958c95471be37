#!/bin/bash
# Overlap trace of crsd_spmv_dist with 2 and 4 ranks on cuda:0 under CUDA MPS.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/overlap
mkdir -p $O
MPS=$(command -v nvidia-cuda-mps-control)
export CUDA_MPS_PIPE_DIRECTORY=/tmp/crsd_mps_pipe CUDA_MPS_LOG_DIRECTORY=/tmp/crsd_mps_log
mkdir -p $CUDA_MPS_PIPE_DIRECTORY $CUDA_MPS_LOG_DIRECTORY
$MPS -d > $O/mps.log 2>&1
sleep 2
for cfg in ${OV_CFGS:-c2:2:direct c2:2:mailbox c5:2:direct c2:4:direct}; do
  IFS=: read c n m <<< "$cfg"
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2977$n scripts/overlap_trace.py $c $m > $O/summary_${c}_${n}_${m}.jsonl 2> $O/err_${c}_${n}_${m}.txt
  echo "$cfg rc=$?" >> $O/mps.log
done
# the same under MPS: bench lines (functional, ranks share one HBM)
for n in 2 4; do
  timeout 600 python bench.py --gpus $n --share-gpu --transport p2p --config c2 --steps 100 --warmup 10 > $O/bench_c2_share$n.json 2> $O/bench_c2_share$n.err
done
echo quit | $MPS >> $O/mps.log 2>&1
echo done
