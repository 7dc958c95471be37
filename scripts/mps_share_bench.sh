#!/bin/bash
# Multi-rank bench with every rank on cuda:0 under CUDA MPS (if the box has
# it): the ranks' kernels then run concurrently instead of time-sliced, so the
# N-rank line shows what row partitioning + the peer-memory halo exchange cost
# when the ranks share one GPU's HBM (total work fixed per rank: weak). Output
# in gpurun_out/.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
MPS=$(command -v nvidia-cuda-mps-control)
echo "mps control: ${MPS:-none}" > gpurun_out/mps.log
if [ -z "$MPS" ]; then exit 0; fi
export CUDA_MPS_PIPE_DIRECTORY=/tmp/crsd_mps_pipe CUDA_MPS_LOG_DIRECTORY=/tmp/crsd_mps_log
mkdir -p $CUDA_MPS_PIPE_DIRECTORY $CUDA_MPS_LOG_DIRECTORY
$MPS -d >> gpurun_out/mps.log 2>&1
sleep 2
for N in ${MPS_NS:-1 2 4}; do
  if [ "$N" = 1 ]; then
    timeout 300 python bench.py --config c2 --steps 100 --warmup 10 --no-cpu ${MPS_ARGS} > gpurun_out/bench_mps1.json 2> gpurun_out/bench_mps1.err
  else
    timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 --master-port 2966$N bench.py --gpus $N --share-gpu --config c2 --steps 100 --warmup 10 --no-cpu ${MPS_ARGS} > gpurun_out/bench_mps$N.json 2> gpurun_out/bench_mps$N.err
  fi
  echo "N=$N rc=$?" >> gpurun_out/mps.log
done
echo quit | $MPS >> gpurun_out/mps.log 2>&1
cat $CUDA_MPS_LOG_DIRECTORY/control.log >> gpurun_out/mps.log 2>/dev/null
