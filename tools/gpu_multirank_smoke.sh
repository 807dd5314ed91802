#!/bin/bash
# The multi-rank bench path (torchrun, gloo coordination, max-over-ranks timing, JSON
# line) exercised on a 1-GPU box: ranks share the GPU with SM-limited dispatchers.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for n in 2 4; do
  STRINGS_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n \
      --master-addr 127.0.0.1 --master-port $((29500 + n)) bench.py --gpus $n --steps 3 --warmup 3 --no-kernels \
      > gpurun_out/multirank_$n.log 2>&1
  echo "n=$n exit $?" >> gpurun_out/multirank_$n.log
done
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29510 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/multirank_ref.log 2>&1
echo "ref exit $?" >> gpurun_out/multirank_ref.log
