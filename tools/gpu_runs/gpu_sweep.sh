#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/sweep.jsonl
for cfg in "--awake-budget 4" "--awake-budget 6" "--awake-budget 8 --admit-cap 16" "--awake-budget 8 --admit-cap 8" "--partitions 4" "--awake-budget 12 --admit-cap 16 --partitions 4" "--device-policy 0" "--device-policy 1" "--balancer 1" "--balancer 6"; do
  echo "== $cfg" >> gpurun_out/sweep.log
  timeout 300 python bench.py --no-static --no-kernels --no-e2e --steps 5 --warmup 2 $cfg > gpurun_out/sw.out 2>> gpurun_out/sweep.log
  python -c "
import json,sys; d=json.loads(open('gpurun_out/sw.out').readline())
print(json.dumps({'args': sys.argv[1], 'value': d['value'], 'frac': d['roofline']['frac'], 'jain': d['jain'], 'cfg': {k: d['config'][k] for k in ('partitions','awake_budget','admit_cap')}}))" "$cfg" >> gpurun_out/sweep.jsonl
done
cat gpurun_out/sweep.jsonl
