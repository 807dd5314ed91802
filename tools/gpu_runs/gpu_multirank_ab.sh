#!/bin/bash
# Shared-GPU multi-rank bench (test mode) with and without the copy partition.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for cc in 0 4 0 4; do
  STRINGS_COPY_CTAS=$cc STRINGS_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
      --master-addr 127.0.0.1 --master-port 29502 bench.py --gpus 2 --steps 3 --warmup 3 --no-kernels --no-e2e \
      > gpurun_out/mr_ab.log 2>&1
  echo "copy_ctas=$cc exit $?"; grep "^{" gpurun_out/mr_ab.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['frac'])"
done
