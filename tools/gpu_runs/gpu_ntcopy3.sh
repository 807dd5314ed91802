#!/bin/bash
# NT staging loops (SSE2 / AVX2 / AVX-512) x copy-thread count: host probe, pageable tests per loop, e2e A/B.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
g++ -O2 -pthread -o /tmp/ntprobe tools/host_ntcopy_probe.cpp && timeout 300 /tmp/ntprobe > gpurun_out/ntprobe3.jsonl 2>&1
for nt in 1 2 3; do
  STRINGS_NT_COPY=$nt timeout 300 python -m pytest tests -m gpu -q -k "pageable" > gpurun_out/nt3_tests_$nt.log 2>&1; echo "tests exit $?" >> gpurun_out/nt3_tests_$nt.log
done
for r in 1 2; do
  for cfg in "1 12" "3 12" "3 14" "3 16"; do
    set -- $cfg
    STRINGS_NT_COPY=$1 STRINGS_COPY_THREADS=$2 timeout 600 python bench.py --no-static --no-kernels > gpurun_out/nt3_bench_$1_$2_$r.log 2>&1
  done
done
cat gpurun_out/ntprobe3.jsonl; tail -n1 gpurun_out/nt3_tests_*.log
for f in gpurun_out/nt3_bench_*.log; do echo $f; python - "$f" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); print(d['value'], d.get('e2e',{}).get('value'), d['roofline']['frac'])
PY
done
