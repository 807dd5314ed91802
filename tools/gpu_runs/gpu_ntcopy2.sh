#!/bin/bash
# PMT staging NT stores: misaligned/ragged pageable test + 4 alternating e2e A/B pairs.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -q -k "pageable" > gpurun_out/nt_tests.log 2>&1; echo "tests exit $?" >> gpurun_out/nt_tests.log
for r in 1 2 3 4; do
  for nt in 1 0; do
    STRINGS_NT_COPY=$nt timeout 600 python bench.py --no-static --no-kernels > gpurun_out/nt2_bench_${nt}_$r.log 2>&1
  done
done
tail -2 gpurun_out/nt_tests.log
for f in gpurun_out/nt2_bench_*.log; do echo $f; python - "$f" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); print(d['value'], d.get('e2e',{}).get('value'), d['roofline']['frac'])
PY
done
