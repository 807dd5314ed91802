#!/bin/bash
# Idle-poll rate of the dispatcher leaders vs copy throughput (C4, 8 logical devices).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -m paper_conf_sc_senguptagsp14_b200.build > /dev/null 2>&1
for pm in 1024 8192 65536; do
  echo "poll_max_ns $pm"
  STRINGS_POLL_MAX_NS=$pm timeout 300 python tools/configs_diag.py C4 --repeats 1 2>&1 | tail -1
done > gpurun_out/diag3.jsonl
STRINGS_KL_MODE_TEST=1 timeout 300 python - >> gpurun_out/diag3.jsonl 2>&1 <<'PY'
print("kl_mode 1 (no persistent kernel)")
import sys; sys.argv=["x","C4","--repeats","1"]
sys.path.insert(0,"tools")
import configs_diag as D, paper_conf_sc_senguptagsp14_b200.strings as S
orig=S.init_from_config
S.init_from_config=lambda cfg, **kw: orig(cfg, kl_mode=1, **kw)
D.main()
PY
cat gpurun_out/diag3.jsonl
