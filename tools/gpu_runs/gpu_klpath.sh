#!/bin/bash
# KL path latency breakdown under load (C1, C3, C2 scaled) with and without the item via the copy ring.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/klpath.jsonl
for v in 0 1; do
  for c in C1 C3; do
    STRINGS_ITEM_VIA_COPY=$v timeout 300 python tools/configs_diag.py $c --repeats 2 | sed "s/^{/{\"item_via_copy\": $v, /" >> gpurun_out/klpath.jsonl 2>&1
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/klpath.jsonl'):
    if not l.startswith('{'): print(l.strip()); continue
    d=json.loads(l)
    print(d['item_via_copy'], d['config'], d['span_ms'], {k: v for k, v in d.items() if k.endswith('kl_path_us_p50')})
PY
