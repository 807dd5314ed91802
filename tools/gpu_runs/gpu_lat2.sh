#!/bin/bash
# KL pickup latency decomposition (calibrated clocks), GPU tests, C2 bench, C4 diag.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -m paper_conf_sc_senguptagsp14_b200.build > /dev/null 2>&1
timeout 300 python tools/latency_probe.py > gpurun_out/lat2.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-static --no-kernels --no-e2e > gpurun_out/bench.log 2>&1
python tools/show_bench.py gpurun_out/bench.log value roofline continuous phase_latency roofline_kernel issue_us_per_job >> gpurun_out/lat2.txt 2>&1
timeout 300 python tools/configs_diag.py C4 --repeats 1 >> gpurun_out/lat2.txt 2>&1
cat gpurun_out/lat2.txt; tail -3 gpurun_out/pytest_gpu.log
