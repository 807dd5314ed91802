#!/bin/bash
# Copy partition: full GPU suite after the ring-index ownership fix, C1 diag A/B, configs A/B.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
STRINGS_STALL_DUMP_S=30 timeout 1200 python -m pytest tests -m gpu -x -q --timeout 300 --timeout-method=thread > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
tail -4 gpurun_out/pytest_gpu.log
for cc in 4 0; do
  for r in 1 2; do
    STRINGS_COPY_CTAS=$cc timeout 300 python tools/configs_diag.py C1 --repeats 3 --trace gpurun_out/c1_trace_cc$cc.txt >> gpurun_out/c1_diag_cc$cc.jsonl 2>&1
  done
  echo "cc=$cc"; cat gpurun_out/c1_diag_cc$cc.jsonl
done
