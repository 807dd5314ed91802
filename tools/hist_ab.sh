#!/bin/bash
# HIST bulk-pipeline threshold A/B on the box: tools/next2_probe.py per build
# (STRINGS_HIST_BULK_MIN_CHUNKS = whole 32 KB chunks per CTA from which the TMA
# bulk pipeline is used; below it the 16-B LDG path).
cd "$(dirname "$0")/.."
for v in ${HIST_AB_VALUES:-1 8 16 40}; do
  STRINGS_NVCC_EXTRA="-DSTRINGS_HIST_BULK_MIN_CHUNKS=$v" python -m paper_conf_sc_senguptagsp14_b200.build >/dev/null 2>&1 || { echo "build failed $v"; continue; }
  echo "== min chunks $v"; timeout 120 python tools/next2_probe.py | grep HIST
done
python -m paper_conf_sc_senguptagsp14_b200.build >/dev/null 2>&1
