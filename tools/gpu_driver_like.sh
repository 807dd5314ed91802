#!/bin/bash
# The round-end driver's sequence on one B200 (build, GPU tests, smoke, bench,
# reference arm, ncu launch list over smoke), logs in gpurun_out/driver_*.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
rm -f paper_conf_sc_senguptagsp14_b200/lib/*.so
timeout 600 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/driver_build.log 2>&1; echo "build rc=$?"
timeout 1500 python -m pytest tests/ -x -q -m gpu > gpurun_out/driver_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/driver_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/driver_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/driver_smoke.log
timeout 1200 python bench.py > gpurun_out/driver_bench.log 2>&1; echo "bench rc=$?"
grep '^{' gpurun_out/driver_bench.log | tail -1 > gpurun_out/driver_bench.json
python tools/show_bench.py gpurun_out/driver_bench.json value ms_per_step e2e speedup_vs_static gpu_launches | cut -c1-200
python -c "import json; d=json.load(open('gpurun_out/driver_bench.json')); r=d['roofline']; print('roofline', r['frac'], r['achieved'], r['duration_us_mean'])"
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/driver_ref.log 2>&1; echo "ref rc=$?"; tail -1 gpurun_out/driver_ref.log | cut -c1-200
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/driver_launches_smoke.csv python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/driver_ncu_smoke.log 2>&1; echo "ncu smoke rc=$?"
