#!/bin/bash
# P = 1 vs P = 2 (with KL slot lending) on C2: throughput and the XFER item (3 alternating pairs).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/p_lend.jsonl
for r in 1 2 3; do
  for cfg in "--partitions 2" "--partitions 1"; do
    timeout 300 python bench.py --no-static --no-kernels --no-e2e $cfg > gpurun_out/pl.out 2>&1
    grep '^{' gpurun_out/pl.out | python -c "
import json,sys; d=json.loads(sys.stdin.read()); rk=d['roofline_kernel']
print(json.dumps({'args': sys.argv[1], 'run': int(sys.argv[2]), 'value': d['value'], 'link_frac': d['roofline']['frac'], 'item_frac': rk['frac'], 'item_body_frac': rk.get('body_only', {}).get('frac'), 'jain': d['jain']}))" "$cfg" $r >> gpurun_out/p_lend.jsonl
  done
done
cat gpurun_out/p_lend.jsonl
