#!/bin/bash
# KL work items through the copy partition for copy-engine jobs: GPU suite + configs + bench.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
STRINGS_STALL_DUMP_S=30 timeout 1200 python -m pytest tests -m gpu -x -q --timeout 300 --timeout-method=thread > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
tail -4 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --configs --config-repeats 3 > gpurun_out/smc3_configs.jsonl 2>&1
python - gpurun_out/smc3_configs.jsonl <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l)
        if 'config' in d: print(d['config'], d['jobs_per_s'], d['span_ms'], d['span_ms_min_max'], d['roofline_frac'], d.get('sm_copy_ops'), d['status'])
PY
timeout 600 python bench.py > gpurun_out/smc3_bench.log 2>&1
python - gpurun_out/smc3_bench.log <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); print(d['value'], d['e2e']['value'], d['roofline']['frac'], d.get('sm_copy_ops_per_step'), d['jain'], d.get('speedup_vs_static'))
PY
