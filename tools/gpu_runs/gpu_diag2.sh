#!/bin/bash
# Copy-stream concurrency on one B200 + shared vs per-logical copy streams.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -m paper_conf_sc_senguptagsp14_b200.build > /dev/null 2>&1
timeout 300 python tools/copy_concurrency.py > gpurun_out/copy_conc.jsonl 2>&1
for a in "C4" "C5" "C3" "C1"; do
  STRINGS_COPY_STREAMS=physical timeout 300 python tools/configs_diag.py $a 2>&1 | tail -1
done > gpurun_out/diag2.jsonl
cat gpurun_out/copy_conc.jsonl gpurun_out/diag2.jsonl
