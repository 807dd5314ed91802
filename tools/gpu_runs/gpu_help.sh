#!/bin/bash
# KL slot lending (an idle sibling partition joins VSCALE/XFER items): tests, fuzz, bench A/B.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
STRINGS_STALL_DUMP_S=20 timeout 900 python -m pytest tests -m gpu -x -q --timeout 120 --timeout-method=thread > gpurun_out/pytest_help.log 2>&1; echo "pytest exit $? $(tail -1 gpurun_out/pytest_help.log)"
STRINGS_STALL_DUMP_S=20 timeout 600 python tests/fuzz_gpu.py 5000 300 | tail -2
for v in 1 0; do
  STRINGS_KL_HELP=$v timeout 600 python bench.py --no-static > gpurun_out/help_bench_$v.log 2>&1
  grep '^{' gpurun_out/help_bench_$v.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); rk=d['roofline_kernel']; print('help=$v', d['value'], d['roofline']['frac'], rk['frac'], rk.get('body_only'), d['phase_latency']['XFER'], d['phase_latency']['GEMM'])"
done
