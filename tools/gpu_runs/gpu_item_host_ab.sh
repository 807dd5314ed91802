#!/bin/bash
# A/B: non-GEMM KL items read by the leader from host-mapped staging (1) vs DMA'd by the copy engine (0).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/item_host_ab.jsonl
STRINGS_ITEM_FROM_HOST=1 timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 --timeout-method=thread > gpurun_out/pt_ih.log 2>&1; echo "pytest (item from host) exit $? $(tail -1 gpurun_out/pt_ih.log)"
for r in 1 2; do
  for v in 1 0; do
    STRINGS_ITEM_FROM_HOST=$v BENCH_CONFIGS=C1,C3,C4,C2 timeout 900 python bench.py --configs --config-repeats 3 > gpurun_out/ih.log 2>&1
    python - gpurun_out/ih.log $v $r >> gpurun_out/item_host_ab.jsonl <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l)
        if 'config' in d:
            print(json.dumps({"item_from_host": int(sys.argv[2]), "run": int(sys.argv[3]), **{k: d[k] for k in ("config","jobs_per_s","span_ms","span_ms_min_max","roofline_frac","tstar_ms","status")}}))
PY
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/item_host_ab.jsonl'):
    d=json.loads(l); print(d['item_from_host'], d['run'], d['config'], d['span_ms'], d['span_ms_min_max'], d['roofline_frac'])
PY
for v in 1 0; do STRINGS_ITEM_FROM_HOST=$v timeout 600 python bench.py --no-static --no-kernels > gpurun_out/ihb$v.log 2>&1; grep '^{' gpurun_out/ihb$v.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bench item_from_host=$v', d['value'], d['roofline']['frac'], d['phase_latency']['XFER'])"; done
