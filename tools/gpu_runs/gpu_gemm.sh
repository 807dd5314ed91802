#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -k gemm --timeout 300 --timeout-method=thread > gpurun_out/pytest_gemm.log 2>&1; tail -1 gpurun_out/pytest_gemm.log
timeout 600 python bench.py --no-static --no-e2e --steps 5 > gpurun_out/bench.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').readline()); print(d['value'], d['roofline']['frac'], json.dumps(d['phase_latency']), json.dumps(d['kernel_rooflines']))"
timeout 300 ncu --set full --clock-control none --import-source on -k regex:oneshot -s 1 -c 1 -o gpurun_out/prof_gemm python tools/kernel_probe.py gemm > gpurun_out/ncu_gemm.log 2>&1
