#!/bin/bash
# Streaming pipeline after the stage-reuse fix: (stages, chunk KB, load lead) sweep.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/stream_lead.jsonl
cp /dev/null gpurun_out/stream_lead2.jsonl
for v in "6 32 4" "7 32 5" "7 32 4" "6 36 4" "4 56 2"; do
  set -- $v
  export STRINGS_NVCC_EXTRA="-DSTRINGS_STREAM_STAGES=$1 -DSTRINGS_STREAM_CHUNK_KB=$2 -DSTRINGS_STREAM_LEAD=$3"
  python -m paper_conf_sc_senguptagsp14_b200.build --force > /dev/null 2>&1 || { echo "{\"build_failed\": \"$v\"}" >> gpurun_out/stream_lead.jsonl; continue; }
  PROBE_QUICK=1 timeout 120 python tools/partition_probe.py | sed "s/^{/{\"lead_variant\": \"$v\", /" >> gpurun_out/stream_lead.jsonl 2>&1
  timeout 120 python -c "
import json, torch, bench
from paper_conf_sc_senguptagsp14_b200 import strings as S
r = bench.kernel_rooflines(torch, S, bench.measured_peaks())
print(json.dumps({'lead_variant': '$v', 'full_gpu': [(x['kernel'], x.get('ctas'), x['achieved'], x['frac']) for x in r]}))
" >> gpurun_out/stream_lead.jsonl 2>&1
done
unset STRINGS_NVCC_EXTRA
python -m paper_conf_sc_senguptagsp14_b200.build --force > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x > gpurun_out/kernels_tests.log 2>&1; tail -1 gpurun_out/kernels_tests.log
cat gpurun_out/stream_lead.jsonl
