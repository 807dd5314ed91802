#!/bin/bash
# Round confirmation: smoke, GPU tests, default bench line, latency probe, all configs measured.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
NCU=0 bash tools/gpu_round.sh > gpurun_out/round.txt 2>&1
timeout 300 python tools/latency_probe.py > gpurun_out/latency.json 2>&1
timeout 1500 python bench.py --configs > gpurun_out/configs.jsonl 2>gpurun_out/configs.err
tail -6 gpurun_out/round.txt; cat gpurun_out/latency.json; cut -c1-400 gpurun_out/configs.jsonl; tail -3 gpurun_out/configs.err
