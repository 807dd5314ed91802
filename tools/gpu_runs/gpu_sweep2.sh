#!/bin/bash
# C2 A/M/P sweep with the copy partition (2 passes, alternating).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/sweep2.jsonl
for r in 1 2; do
for cfg in "--awake-budget 4" "--awake-budget 3 --admit-cap 6" "--awake-budget 6 --admit-cap 12" "--awake-budget 8 --admit-cap 16" "--partitions 1 --awake-budget 3 --admit-cap 6" "--partitions 1"; do
  timeout 300 python bench.py --no-static --no-kernels --no-e2e --steps 6 --warmup 3 $cfg > gpurun_out/sw.out 2>> gpurun_out/sweep2.log
  python -c "
import json,sys; d=json.loads(open('gpurun_out/sw.out').readline())
print(json.dumps({'args': sys.argv[1], 'run': int(sys.argv[2]), 'value': d['value'], 'frac': d['roofline']['frac'], 'continuous_frac': d['continuous']['frac_host_link'], 'jain': d['jain'], 'xfer_item_frac': d['roofline_kernel']['frac'], 'xfer_body_frac': d['roofline_kernel'].get('body_only', {}).get('frac'), 'cfg': {k: d['config'][k] for k in ('partitions','awake_budget','admit_cap')}}))" "$cfg" $r >> gpurun_out/sweep2.jsonl
done
done
cat gpurun_out/sweep2.jsonl
