#!/bin/bash
# Evidence run: bench line, ncu launch list (kl-mode 1), ncu --set full of each tenant kernel, latency probe.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python bench.py > gpurun_out/bench.log 2>&1; echo "bench exit $?" >> gpurun_out/bench.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --kl-mode 1 --steps 2 --warmup 1 --no-static --no-e2e > gpurun_out/bench_ncu.log 2>&1
for k in vscale xfer gemm; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:oneshot -s 1 -c 1 \
      -o gpurun_out/prof_$k python tools/kernel_probe.py $k > gpurun_out/ncu_$k.log 2>&1
done
timeout 120 python tools/latency_probe.py > gpurun_out/latency.json 2>&1
tail -2 gpurun_out/bench.log | cut -c1-400
