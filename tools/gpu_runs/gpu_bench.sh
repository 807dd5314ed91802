#!/bin/bash
# One gpurun call: remaining GPU tests, bench line, ncu launch list, ncu full captures.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_scheduler.py -q --timeout 600 --timeout-method=thread --durations=20 \
    -k "pageable or full_size or measured" > gpurun_out/pytest_gpu2.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu2.log
timeout 1200 python bench.py > gpurun_out/bench.log 2>&1; echo "bench exit $?" >> gpurun_out/bench.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --kl-mode 1 --steps 2 --warmup 1 --no-static --no-e2e > gpurun_out/bench_ncu.log 2>&1; echo "ncu list exit $?" >> gpurun_out/bench_ncu.log
for k in vscale xfer gemm; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:oneshot -s 1 -c 1 \
      -o gpurun_out/prof_$k python tools/kernel_probe.py $k > gpurun_out/ncu_$k.log 2>&1; echo "ncu $k exit $?" >> gpurun_out/ncu_$k.log
done
tail -3 gpurun_out/pytest_gpu2.log; tail -3 gpurun_out/bench.log; tail -2 gpurun_out/bench_ncu.log
