#!/bin/bash
# Copy partition sweep: CTAs x size threshold on the small-copy configs (C1, C3) and C4/C5/C2.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
rm -f gpurun_out/smc_sweep.jsonl
for cfg in "4 1048576" "8 1048576" "16 1048576" "8 4194304" "16 4194304" "32 4194304"; do
  set -- $cfg
  STRINGS_COPY_CTAS=$1 STRINGS_SM_COPY_MAX=$2 BENCH_CONFIGS=C1,C3,C4,C5,C2 timeout 900 python bench.py --configs --config-repeats 3 > gpurun_out/smc_sw.log 2>&1
  python - gpurun_out/smc_sw.log $1 $2 >> gpurun_out/smc_sweep.jsonl <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l)
        if 'config' in d:
            print(json.dumps({"copy_ctas": int(sys.argv[2]), "sm_copy_max": int(sys.argv[3]), **{k: d[k] for k in ("config","jobs_per_s","span_ms","span_ms_min_max","roofline_frac","tstar_ms","sm_copy_ops","status")}}))
PY
done
python - <<'PY'
import json
for l in open('gpurun_out/smc_sweep.jsonl'):
    d=json.loads(l); print(d['copy_ctas'], d['sm_copy_max'], d['config'], d['span_ms'], d['span_ms_min_max'], d['roofline_frac'], d['sm_copy_ops'], d['status'])
PY
