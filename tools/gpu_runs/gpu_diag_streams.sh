#!/bin/bash
# C4/C5 (8 logical devices on one B200): per-logical vs shared physical copy streams.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for a in C4 C5 C1; do
  for mode in logical physical logical physical; do
    STRINGS_COPY_STREAMS=$mode timeout 300 python tools/configs_diag.py $a --repeats 2 2>&1 | tail -1 | sed "s/^{/{\"streams\": \"$mode\", /"
  done
done > gpurun_out/diag_streams.jsonl
