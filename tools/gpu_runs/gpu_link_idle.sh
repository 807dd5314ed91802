#!/bin/bash
# Host-link behaviour after idle + C1 trace (logical / physical copy streams) for gap analysis.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python tools/link_idle_probe.py > gpurun_out/link_idle.jsonl 2>&1
timeout 300 python tools/configs_diag.py C1 --repeats 3 --trace gpurun_out/c1_trace_logical.txt > gpurun_out/c1_diag.jsonl 2>&1
STRINGS_COPY_STREAMS=physical timeout 300 python tools/configs_diag.py C1 --repeats 3 --trace gpurun_out/c1_trace_physical.txt >> gpurun_out/c1_diag.jsonl 2>&1
cat gpurun_out/link_idle.jsonl gpurun_out/c1_diag.jsonl
