#!/bin/bash
# Multi-logical-device configs: where the span goes (tools/configs_diag.py).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -m paper_conf_sc_senguptagsp14_b200.build > /dev/null 2>&1
for a in "C1" "C3" "C4" "C5" "C4 --policy PS" "C4 --gpus 1" "C5 --gpus 1" "C3 --gpus 1" "C1 --gpus 1"; do
  timeout 300 python tools/configs_diag.py $a 2>&1 | tail -1
done > gpurun_out/diag.jsonl
cat gpurun_out/diag.jsonl
