#!/bin/bash
# Device-memory vs host-memory KL doorbell: KL latency, C2 bench, C4 (8 logical devices).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -m paper_conf_sc_senguptagsp14_b200.build > /dev/null 2>&1
for db in device host; do
  echo "doorbell $db"
  STRINGS_DOORBELL=$db timeout 300 python tools/latency_probe.py 2>&1 | tail -1
  STRINGS_DOORBELL=$db timeout 600 python bench.py --no-static --no-kernels --no-e2e > gpurun_out/bench_$db.log 2>&1
  python tools/show_bench.py gpurun_out/bench_$db.log value roofline continuous phase_latency decision_us_per_job issue_us_per_job 2>&1
  STRINGS_DOORBELL=$db timeout 300 python tools/configs_diag.py C4 --repeats 1 2>&1 | tail -1
  STRINGS_DOORBELL=$db timeout 300 python tools/configs_diag.py C1 --repeats 2 2>&1 | tail -1
done > gpurun_out/doorbell.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
cat gpurun_out/doorbell.txt; tail -2 gpurun_out/pytest_gpu.log
