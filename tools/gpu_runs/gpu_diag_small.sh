#!/bin/bash
# Small-copy configs (C1, C3) on one B200: per-logical vs shared physical copy streams.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for a in C1 C3; do
  for mode in logical physical; do
    for r in 1 2; do
      STRINGS_COPY_STREAMS=$mode timeout 300 python tools/configs_diag.py $a --repeats 3 2>&1 | tail -1 | sed "s/^{/{\"streams\": \"$mode\", /"
    done
  done
done > gpurun_out/diag_small.jsonl
cut -c1-600 gpurun_out/diag_small.jsonl
