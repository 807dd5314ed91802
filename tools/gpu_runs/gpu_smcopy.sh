#!/bin/bash
# Copy partition (small H2D/D2H as zero-copy SM copies): GPU tests, configs C1/C3 A/B, bench.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/smoke.log
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 --timeout-method=thread > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/smoke.log; tail -15 gpurun_out/pytest_gpu.log
for cc in 4 0; do
  STRINGS_COPY_CTAS=$cc timeout 900 python bench.py --configs --config-repeats 3 > gpurun_out/smc_configs_$cc.jsonl 2>&1
  echo "copy_ctas=$cc"; python - gpurun_out/smc_configs_$cc.jsonl <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l)
        if 'config' in d: print(d['config'], d['jobs_per_s'], d['span_ms'], d['roofline_frac'], d.get('sm_copy_ops'), d['status'])
PY
done
for cc in 4 0; do
  STRINGS_COPY_CTAS=$cc timeout 600 python bench.py --no-static > gpurun_out/smc_bench_$cc.log 2>&1
  echo "bench copy_ctas=$cc"; python - gpurun_out/smc_bench_$cc.log <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); print(d['value'], d['e2e']['value'], d['roofline']['frac'], d.get('sm_copy_ops_per_step'), d['jain'])
PY
done
