#!/bin/bash
# e2e A/B: SSE2 vs AVX2 non-temporal staging loops (3 alternating pairs, 12 copy threads).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for r in 1 2 3; do
  for nt in 1 2; do
    STRINGS_NT_COPY=$nt timeout 600 python bench.py --no-static --no-kernels > gpurun_out/nt4_bench_${nt}_$r.log 2>&1
  done
done
for f in gpurun_out/nt4_bench_*.log; do echo $f; python - "$f" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); print(d['value'], d.get('e2e',{}).get('value'), d['roofline']['frac'])
PY
done
