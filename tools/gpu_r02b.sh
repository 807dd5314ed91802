#!/bin/bash
# Round-2 (second session) confirmation run on one B200: build, GPU test tier,
# GPU fuzz (random workloads, both timing modes, incl. HIST/SCAN/SORT items),
# the bench line, the five configs, the NEXT-2 kernel probe.  Logs in gpurun_out/.
set -u
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -m paper_conf_sc_senguptagsp14_b200.build > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -20 gpurun_out/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
for task in "$@"; do
  case "$task" in
    tests) timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/pytest_gpu.log ;;
    fuzz) timeout 900 python tests/fuzz_gpu.py ${FUZZ_FIRST:-5000} ${FUZZ_COUNT:-150} > gpurun_out/fuzz.log 2>&1; echo "fuzz rc=$?"; tail -3 gpurun_out/fuzz.log ;;
    fuzzbig) timeout 900 python tests/fuzz_gpu.py ${FUZZ_FIRST:-7000} ${FUZZ_COUNT:-40} big > gpurun_out/fuzzbig.log 2>&1; echo "fuzzbig rc=$?"; tail -3 gpurun_out/fuzzbig.log ;;
    bench) timeout 1200 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?"; grep "^{" gpurun_out/bench.log | tail -1 > gpurun_out/bench.json; python tools/show_bench.py gpurun_out/bench.json value ms_per_step roofline e2e speedup_vs_static clocks | cut -c1-300 ;;
    configs) BENCH_CONFIGS=${CONFIGS:-C1,C2,C3,C4,C5} timeout 2400 python bench.py --configs --config-repeats ${REPEATS:-3} > gpurun_out/configs.log 2>&1; echo "configs rc=$?"; grep '^{' gpurun_out/configs.log | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    if 'config' in d: print(d['config'], d.get('jobs_per_s'), d.get('span_ms'), d.get('roofline_frac'))
" ;;
    next2) timeout 300 python tools/next2_probe.py > gpurun_out/next2.log 2>&1; echo "next2 rc=$?"; cat gpurun_out/next2.log ;;
    *) echo "unknown task $task" ;;
  esac
done
