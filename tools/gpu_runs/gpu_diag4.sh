#!/bin/bash
# Small-copy configs (C1, C3): physical copy rates at 4 MiB / 256 KiB and scheduler variants.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -m paper_conf_sc_senguptagsp14_b200.build > /dev/null 2>&1
timeout 300 python tools/copy_concurrency.py > gpurun_out/copy_conc2.jsonl 2>&1
for a in "C1" "C1 --gpus 1" "C3" "C3 --gpus 1" "C3 --awake-budget 8" "C1 --awake-budget 8"; do
  echo "$a"
  timeout 300 python tools/configs_diag.py $a --repeats 3 2>&1 | tail -1
done > gpurun_out/diag4.txt 2>&1
cat gpurun_out/copy_conc2.jsonl gpurun_out/diag4.txt
