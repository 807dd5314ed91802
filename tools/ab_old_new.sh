#!/bin/bash
# Same-box A/B of the C2 bench line between an older commit and the working tree.
# Here:   rm -rf ab_old && mkdir ab_old && git archive <commit> | tar -x -C ab_old
# Box:    /usr/local/graft/bin/gpurun -- 'bash tools/ab_old_new.sh'
# Builds both .so files, then alternates short bench runs (10 steps) old / new x 4;
# AB_CONFIGS=C1,C3 alternates `bench.py --configs` runs of those configs instead.
set -u
cd "$(dirname "$0")/.."
(cd ab_old && python -m paper_conf_sc_senguptagsp14_b200.build > /dev/null 2>&1) || echo old build failed
python -m paper_conf_sc_senguptagsp14_b200.build > /dev/null 2>&1 || echo new build failed
for rep in 1 2 3 4; do
  for v in old new; do
    d=.; [ $v = old ] && d=ab_old
    if [ -n "${AB_CONFIGS:-}" ]; then
      (cd $d && BENCH_CONFIGS=$AB_CONFIGS timeout 900 python bench.py --configs --config-repeats 5 2>/dev/null) | grep '^{' | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    if isinstance(d.get('config'),str): print('$v', d['config'], d['jobs_per_s'], d['span_ms'], d['span_ms_min_max'], d['roofline_frac'], 'dec', d['decision_us_per_job'], 'iss', d['issue_us_per_job'])
"
      continue
    fi
    (cd $d && timeout 300 python bench.py --steps 10 --warmup 3 --no-static --no-e2e --no-kernels 2>/dev/null) | grep '^{' | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); x=d['phase_latency']['XFER']; g=d['phase_latency']['GEMM']
    print('$v', d['value'], d['ms_per_step'], 'item', x['kl_device_us_mean'], 'gemm', g['kl_device_us_mean'], 'frac', d['roofline']['frac'], 'dec', d['decision_us_per_job'], 'iss', d['issue_us_per_job'])
"
  done
done
