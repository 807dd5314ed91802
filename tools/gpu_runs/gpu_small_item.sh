#!/bin/bash
# Small stream items: pipeline vs LDG path (STRINGS_STREAM_MIN_CHUNKS) on 18/36/72 CTAs.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/small_item.jsonl
for m in 0 2 4 8; do
  export STRINGS_NVCC_EXTRA="-DSTRINGS_STREAM_MIN_CHUNKS=$m"
  python -m paper_conf_sc_senguptagsp14_b200.build --force > /dev/null 2>&1 || { echo "{\"build_failed\": $m}" >> gpurun_out/small_item.jsonl; continue; }
  timeout 120 python tools/small_item_probe.py "min_chunks=$m" >> gpurun_out/small_item.jsonl 2>&1
done
unset STRINGS_NVCC_EXTRA
python -m paper_conf_sc_senguptagsp14_b200.build --force > /dev/null 2>&1
python - <<'PY'
import json, collections
rows = [json.loads(l) for l in open('gpurun_out/small_item.jsonl') if l.startswith('{"build"')]
t = collections.defaultdict(dict)
for r in rows: t[(r['kernel'], r['n'], r['ctas'])][r['build']] = r['us']
for k, v in sorted(t.items()): print(k, v)
PY
