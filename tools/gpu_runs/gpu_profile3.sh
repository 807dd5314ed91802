#!/bin/bash
# ncu --set full of the NEXT-2 bodies (HIST, SCAN, SORT) after their rework.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for k in hist scan sort; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:oneshot -s 1 -c 1 \
      -o gpurun_out/prof_$k -f python tools/kernel_probe.py $k > gpurun_out/ncu_$k.log 2>&1
  echo "ncu $k exit $?"
done
