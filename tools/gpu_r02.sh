#!/bin/bash
# Round-2 GPU session helper: `tools/gpu_r02.sh <task> ...` runs on the B200 box
# under gpurun (cwd = repo snapshot).  Logs land in gpurun_out/.
set -u
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
python -m paper_conf_sc_senguptagsp14_b200.build > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
for task in "$@"; do
  case "$task" in
    tests)  timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "tests rc=$?"; tail -5 gpurun_out/pytest_gpu.log ;;
    smoke)  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log ;;
    ncu_smoke) timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_smoke.csv python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/ncu_smoke.log 2>&1; echo "ncu_smoke rc=$?"; tail -3 gpurun_out/ncu_smoke.log; grep -c '"gpu__time_duration.sum"' gpurun_out/launches_smoke.csv ;;
    bench1) timeout 1200 python bench.py --steps ${STEPS:-10} --warmup ${WARMUP:-3} > gpurun_out/bench1.log 2>&1; echo "bench1 rc=$?"; tail -c 3000 gpurun_out/bench1.log ;;
    bench2) timeout 1500 python bench.py --gpus 2 --steps ${STEPS:-5} --warmup ${WARMUP:-3} > gpurun_out/bench2.log 2>&1; echo "bench2 rc=$?"; tail -c 3000 gpurun_out/bench2.log ;;
    bench2tr) timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps ${STEPS:-3} --warmup 3 --no-static --no-baseline-config --no-e2e > gpurun_out/bench2tr.log 2>&1; echo "bench2tr rc=$?"; tail -c 2000 gpurun_out/bench2tr.log ;;
    configs) BENCH_CONFIGS=${CONFIGS:-C1,C2,C3,C4,C5} timeout 2400 python bench.py --configs --config-repeats ${REPEATS:-3} > gpurun_out/configs.log 2>&1; echo "configs rc=$?"; tail -c 4000 gpurun_out/configs.log ;;
    ncu_item) timeout 900 ncu --set full --clock-control none --import-source on -k regex:oneshot -c 4 -f -o gpurun_out/prof_xfer_item python tools/kernel_probe.py xfer_item > gpurun_out/ncu_item.log 2>&1; echo "ncu_item rc=$?"; tail -3 gpurun_out/ncu_item.log ;;
    ncu_launches) timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 1 --no-static --no-e2e --no-kernels > gpurun_out/ncu_launches.log 2>&1; echo "ncu_launches rc=$?"; tail -c 600 gpurun_out/ncu_launches.log ;;
    openloop) timeout 1800 python bench.py --open-loop --open-loop-config ${OLCFG:-C4} > gpurun_out/openloop_${OLCFG:-C4}.log 2>&1; echo "openloop rc=$?"; tail -c 1500 gpurun_out/openloop_${OLCFG:-C4}.log ;;
    configs_ab) for e in 1 0 1 0; do STRINGS_EAGER=$e BENCH_CONFIGS=${CONFIGS:-C1,C3} timeout 1200 python bench.py --configs --config-repeats ${REPEATS:-3} > gpurun_out/configs_eager$e.log 2>&1; echo "eager=$e rc=$?"; python -c "
import json,sys
for l in open('gpurun_out/configs_eager$e.log'):
    if l.startswith('{'):
        d=json.loads(l); print(d['config'], d['jobs_per_s'], d['span_ms'], d['roofline_frac'], d.get('frac_vs_copy_replay'), d['span_ms_min_max'])
"; done ;;
    ncu_kernels) for k in vscale xfer gemm scan hist sort; do timeout 900 ncu --set full --clock-control none --import-source on -k regex:oneshot -c 2 -f -o gpurun_out/prof_$k python tools/kernel_probe.py $k > gpurun_out/ncu_$k.log 2>&1; echo "ncu $k rc=$?"; done ;;
    benchdef) timeout 1200 python bench.py > gpurun_out/benchdef.log 2>&1; echo "benchdef rc=$?"; tail -c 400 gpurun_out/benchdef.log ;;
    ref) timeout 900 python bench.py --impl reference --steps ${STEPS:-20} --warmup ${WARMUP:-5} > gpurun_out/ref.log 2>&1; echo "ref rc=$?"; tail -c 800 gpurun_out/ref.log ;;
    configs_it) for e in 1 0; do STRINGS_ISSUE_THREADS=$e BENCH_CONFIGS=${CONFIGS:-C1,C3,C5,C2} timeout 1800 python bench.py --configs --config-repeats ${REPEATS:-3} > gpurun_out/configs_it$e.log 2>&1; echo "issue_threads=$e rc=$?"; python -c "
import json
for l in open('gpurun_out/configs_it$e.log'):
    if l.startswith('{'):
        d=json.loads(l); print(d['config'], d['jobs_per_s'], d['span_ms'], d['roofline_frac'], d['span_ms_min_max'], 'dec', d['decision_us_per_job'], 'iss', d['issue_us_per_job'])
"; done ;;
    *) echo "unknown task $task" ;;
  esac
done
