#!/bin/bash
# Re-capture after the streaming-pipeline fix: ncu --set full of VSCALE, XFER, the C2 XFER item (74 CTAs),
# GEMM; ncu launch list of bench --kl-mode 1.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for k in vscale xfer xfer_item gemm; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:oneshot -s 1 -c 1 \
      -o gpurun_out/prof_$k -f python tools/kernel_probe.py $k > gpurun_out/ncu_$k.log 2>&1
  echo "ncu $k exit $?"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --kl-mode 1 --steps 2 --warmup 1 --no-static --no-e2e > gpurun_out/bench_ncu.log 2>&1
echo "launch list exit $?"
ls -la gpurun_out/*.ncu-rep
