#!/bin/bash
# A/B: KL work items of copy-engine jobs via the copy partition (1) or the CE DMA (0); configs C1, C3, C4, C2.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
rm -f gpurun_out/item_ab.jsonl
STRINGS_ITEM_VIA_COPY=1 timeout 600 python -m pytest tests -m gpu -x -q -k "small_copies or full_size" --timeout 300 --timeout-method=thread > gpurun_out/pt.log 2>&1; echo "pytest exit $?" >> gpurun_out/pt.log; tail -2 gpurun_out/pt.log
for r in 1 2; do
  for v in 1 0; do
    STRINGS_ITEM_VIA_COPY=$v STRINGS_STALL_DUMP_S=30 BENCH_CONFIGS=C1,C3,C4,C2 timeout 900 python bench.py --configs --config-repeats 3 > gpurun_out/item_ab.log 2>&1
    python - gpurun_out/item_ab.log $v $r >> gpurun_out/item_ab.jsonl <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l)
        if 'config' in d:
            print(json.dumps({"item_via_copy": int(sys.argv[2]), "run": int(sys.argv[3]), **{k: d[k] for k in ("config","jobs_per_s","span_ms","span_ms_min_max","roofline_frac","tstar_ms","sm_copy_ops","status")}}))
PY
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/item_ab.jsonl'):
    d=json.loads(l); print(d['item_via_copy'], d['run'], d['config'], d['span_ms'], d['span_ms_min_max'], d['roofline_frac'], d['tstar_ms'])
PY
