#!/bin/bash
# All configs measured (with copy-only replay floor).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -m paper_conf_sc_senguptagsp14_b200.build > /dev/null 2>&1
timeout 1500 python bench.py --configs > gpurun_out/configs.jsonl 2>gpurun_out/configs.err
python - <<'PY'
import json
for l in open("gpurun_out/configs.jsonl"):
    d = json.loads(l)
    print(d["config"], d["jobs_per_s"], "span", d["span_ms"], "T*", d["tstar_ms"], d["roofline_frac"], "copy-only", d["copy_only_ms"], d["frac_vs_copy_only"])
PY
tail -3 gpurun_out/configs.err
