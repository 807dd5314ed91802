#!/bin/bash
# KL slot lending A/B on the C2 bench (4 alternating pairs) and configs C4/C5 once each.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/help_ab.jsonl
for r in 1 2 3 4; do
  for v in 1 0; do
    STRINGS_KL_HELP=$v timeout 600 python bench.py --no-static --no-e2e > gpurun_out/hab.log 2>&1
    grep '^{' gpurun_out/hab.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); rk=d['roofline_kernel']; print(json.dumps({'kl_help': $v, 'run': $r, 'value': d['value'], 'link_frac': d['roofline']['frac'], 'continuous_frac': d['continuous']['frac_host_link'], 'item_frac': rk['frac'], 'item_body_frac': rk.get('body_only', {}).get('frac'), 'jain': d['jain']}))" >> gpurun_out/help_ab.jsonl
  done
done
cat gpurun_out/help_ab.jsonl
for v in 1 0; do
  STRINGS_KL_HELP=$v BENCH_CONFIGS=C1,C3,C4,C5 timeout 900 python bench.py --configs --config-repeats 2 > gpurun_out/hcfg_$v.log 2>&1
  python - gpurun_out/hcfg_$v.log $v <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l)
        if 'config' in d: print('help', sys.argv[2], d['config'], d['span_ms'], d['roofline_frac'], d['status'])
PY
done
