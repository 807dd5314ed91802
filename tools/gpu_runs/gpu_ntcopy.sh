#!/bin/bash
# PMT staging with non-temporal stores: host probe + bench e2e A/B (STRINGS_NT_COPY=0/1, alternating).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
lscpu > gpurun_out/lscpu.txt 2>&1
g++ -O2 -pthread -o /tmp/ntprobe tools/host_ntcopy_probe.cpp && timeout 300 /tmp/ntprobe > gpurun_out/ntprobe.jsonl 2>&1
timeout 300 python -m pytest tests -m gpu -q -k "pageable or full_size_c2" > gpurun_out/nt_tests.log 2>&1; echo "tests exit $?" >> gpurun_out/nt_tests.log
for r in 1 2; do
  for nt in 0 1; do
    STRINGS_NT_COPY=$nt timeout 600 python bench.py --no-static --no-kernels > gpurun_out/nt_bench_${nt}_$r.log 2>&1
  done
done
cat gpurun_out/ntprobe.jsonl; tail -2 gpurun_out/nt_tests.log
for f in gpurun_out/nt_bench_*.log; do echo $f; python - "$f" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); print(d['value'], d.get('e2e',{}).get('value'), d['roofline']['frac'])
PY
done
