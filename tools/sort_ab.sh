#!/bin/bash
# SORT layout A/B on the box: 8 vs 32 keys per thread (STRINGS_SORT_KPT), the
# kernel tests for SORT, then tools/next2_probe.py's SORT row per build.
cd "$(dirname "$0")/.."
for v in ${SORT_AB_VALUES:-8 32}; do
  STRINGS_NVCC_EXTRA="-DSTRINGS_SORT_KPT=$v" python -m paper_conf_sc_senguptagsp14_b200.build >/dev/null 2>&1 || { echo "build failed $v"; continue; }
  echo "== keys per thread $v"
  timeout 300 python -m pytest tests/test_gpu_kernels.py -m gpu -q -k sort 2>&1 | tail -1
  for i in 1 2; do timeout 120 python tools/next2_probe.py | grep SORT; done
done
python -m paper_conf_sc_senguptagsp14_b200.build >/dev/null 2>&1
