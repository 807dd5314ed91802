#!/bin/bash
# Mixed-size host-link traffic probe (C3 shape): small copies on CE vs SM zero-copy.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mix_probe tools/mix_probe.cu && timeout 120 /tmp/mix_probe 128 > gpurun_out/mix_probe.jsonl 2>&1
timeout 120 /tmp/mix_probe 16 >> gpurun_out/mix_probe.jsonl 2>&1
cat gpurun_out/mix_probe.jsonl
