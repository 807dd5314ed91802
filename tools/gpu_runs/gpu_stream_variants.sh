#!/bin/bash
# Streaming pipeline shape sweep (stages x chunk KB): partition probe at 2^24 + full-GPU 2^28 rooflines.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/stream_variants.jsonl
for v in "4 48" "6 32" "5 40" "8 24" "3 64" "12 16"; do
  set -- $v
  export STRINGS_NVCC_EXTRA="-DSTRINGS_STREAM_STAGES=$1 -DSTRINGS_STREAM_CHUNK_KB=$2"
  python -m paper_conf_sc_senguptagsp14_b200.build --force > /dev/null 2>&1 || { echo "build $v failed" >> gpurun_out/stream_variants.jsonl; continue; }
  PROBE_QUICK=1 timeout 120 python tools/partition_probe.py >> gpurun_out/stream_variants.jsonl 2>&1
  timeout 120 python -c "
import json, torch, bench
from paper_conf_sc_senguptagsp14_b200 import strings as S
r = bench.kernel_rooflines(torch, S, bench.measured_peaks())
print(json.dumps({'variant': '$v', 'full_gpu_2^28': [(x['kernel'], x['achieved'], x['frac']) for x in r]}))
" >> gpurun_out/stream_variants.jsonl 2>&1
done
unset STRINGS_NVCC_EXTRA
python -m paper_conf_sc_senguptagsp14_b200.build --force > /dev/null 2>&1
