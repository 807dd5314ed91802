# C1/C2/C3/C5 at awake budgets A = 4 (default), 6, 8 (M = 2A), MEASURED, median of 3
for a in 4 6 8; do
  BENCH_AWAKE_BUDGET=$a BENCH_CONFIGS=C1,C3,C5,C2 timeout 1500 python bench.py --configs --config-repeats 3 > gpurun_out/asweep_$a.log 2>&1
  python -c "
import json
for l in open('gpurun_out/asweep_$a.log'):
    if l.startswith('{'):
        d=json.loads(l); print('A=$a', d['config'], d['jobs_per_s'], d['span_ms'], d['roofline_frac'], d['span_ms_min_max'])
"
done
