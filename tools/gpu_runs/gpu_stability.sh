#!/bin/bash
# Stability: GPU suite twice, bench three times, configs twice (no hangs, no flakes, spread of the numbers).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/stab.txt
for r in 1 2; do
  STRINGS_STALL_DUMP_S=30 timeout 900 python -m pytest tests -m gpu -q --timeout 300 --timeout-method=thread -p no:randomly > gpurun_out/stab_pytest_$r.log 2>&1
  echo "pytest run $r exit $? $(tail -1 gpurun_out/stab_pytest_$r.log)" >> gpurun_out/stab.txt
done
for r in 1 2 3; do
  timeout 600 python bench.py --no-static > gpurun_out/stab_bench_$r.log 2>&1
  grep '^{' gpurun_out/stab_bench_$r.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bench', d['value'], d['roofline']['frac'], d['continuous']['frac_host_link'], d['e2e']['value'], d['jain'], d['roofline_kernel']['frac'])" >> gpurun_out/stab.txt
done
for r in 1 2; do
  timeout 900 python bench.py --configs > gpurun_out/stab_cfg_$r.jsonl 2>&1
  python - gpurun_out/stab_cfg_$r.jsonl >> gpurun_out/stab.txt <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l)
        if 'config' in d: print('cfg', d['config'], d['jobs_per_s'], d['span_ms'], d['roofline_frac'], d['status'])
PY
done
cat gpurun_out/stab.txt
