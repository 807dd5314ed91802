#!/bin/bash
# quick: GPU scheduler tests + bench (no static, no kernels) with trace
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_scheduler.py -q --timeout 600 --timeout-method=thread -x > gpurun_out/pytest_sched.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_sched.log
timeout 900 python bench.py --no-static --no-kernels --trace-out gpurun_out/c2_trace.txt ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "bench exit $?" >> gpurun_out/bench.log
tail -2 gpurun_out/pytest_sched.log; tail -2 gpurun_out/bench.log | cut -c1-1500
