#!/bin/bash
# Copy partition only while the engine is busy (default) vs always: tests, latency probe, configs, bench.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 --timeout-method=thread -k "small_copies or pageable or full_size_c2 or measured" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $? $(tail -1 gpurun_out/pytest_gpu.log)"
for w in busy always; do
  STRINGS_SM_COPY_WHEN=$w timeout 300 python tools/latency_probe.py > gpurun_out/lat_$w.json 2>&1
  echo "$w latency: $(cat gpurun_out/lat_$w.json | cut -c1-200)"
done
: > gpurun_out/smwhen.jsonl
for r in 1 2; do
  for w in busy always; do
    STRINGS_SM_COPY_WHEN=$w BENCH_CONFIGS=C1,C3,C4,C2 timeout 900 python bench.py --configs --config-repeats 3 > gpurun_out/smw.log 2>&1
    python - gpurun_out/smw.log $w $r >> gpurun_out/smwhen.jsonl <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l)
        if 'config' in d:
            print(json.dumps({"sm_copy_when": sys.argv[2], "run": int(sys.argv[3]), **{k: d[k] for k in ("config","jobs_per_s","span_ms","span_ms_min_max","roofline_frac","tstar_ms","sm_copy_ops","status")}}))
PY
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/smwhen.jsonl'):
    d=json.loads(l); print(d['sm_copy_when'], d['run'], d['config'], d['span_ms'], d['roofline_frac'], d['sm_copy_ops'])
PY
