#!/bin/bash
# A/B with the copy partition on: per-logical-device copy streams vs one H2D + one D2H stream per GPU.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
rm -f gpurun_out/streams_ab.jsonl
for r in 1 2; do
  for v in logical physical; do
    STRINGS_COPY_STREAMS=$v BENCH_CONFIGS=C1,C3,C4,C5 timeout 900 python bench.py --configs --config-repeats 3 > gpurun_out/streams_ab.log 2>&1
    python - gpurun_out/streams_ab.log $v $r >> gpurun_out/streams_ab.jsonl <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l)
        if 'config' in d:
            print(json.dumps({"copy_streams": sys.argv[2], "run": int(sys.argv[3]), **{k: d[k] for k in ("config","jobs_per_s","span_ms","span_ms_min_max","roofline_frac","tstar_ms","sm_copy_ops","status")}}))
PY
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/streams_ab.jsonl'):
    d=json.loads(l); print(d['copy_streams'], d['run'], d['config'], d['span_ms'], d['span_ms_min_max'], d['roofline_frac'], d['tstar_ms'])
PY
