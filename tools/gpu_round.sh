#!/bin/bash
# One gpurun call: smoke, full GPU test tier (with durations), bench line, ncu captures.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 --timeout-method=thread --durations=25 \
    > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
timeout 1200 python bench.py > gpurun_out/bench.log 2>&1; echo "bench exit $?" >> gpurun_out/bench.log
if [ "${NCU:-1}" = "1" ]; then
  for k in ${NCU_KERNELS:-vscale gemm}; do
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:oneshot -s 1 -c 1 \
        -o gpurun_out/prof_$k python tools/kernel_probe.py $k > gpurun_out/ncu_$k.log 2>&1; echo "ncu $k exit $?" >> gpurun_out/ncu_$k.log
  done
fi
tail -3 gpurun_out/smoke.log; tail -32 gpurun_out/pytest_gpu.log; tail -3 gpurun_out/bench.log
