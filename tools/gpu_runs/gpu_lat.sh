#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python tools/latency_probe.py > gpurun_out/latency.json 2>&1
timeout 600 python bench.py --no-static --no-kernels --no-e2e --trace-out gpurun_out/c2_trace.txt > gpurun_out/bench.log 2>&1
cat gpurun_out/latency.json; python -c "
import json; d=json.loads(open('gpurun_out/bench.log').readline()); print(d['value'], d['roofline']['frac'], json.dumps(d['phase_latency']))"
