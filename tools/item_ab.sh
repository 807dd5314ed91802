#!/bin/bash
# C2 XFER work-item latency A/B on the box: bench.py (short, no static / e2e /
# kernel legs) per build variant; prints the item's device time (claim -> last
# CTA), its body (t_exec -> end) and the roofline fraction.  Variants are
# STRINGS_NVCC_EXTRA flag sets separated by ';' (',' inside a set = space).
cd "$(dirname "$0")/.."
IFS=';' read -ra VARS <<< "${ITEM_AB_VARIANTS:--DSTRINGS_TEXEC_FIRST;-DSTRINGS_TEXEC_FIRST,-DSTRINGS_GEN_SPIN}"
for rep in 1 2; do
for v in "${VARS[@]}"; do
  STRINGS_NVCC_EXTRA="${v//,/ }" python -m paper_conf_sc_senguptagsp14_b200.build >/dev/null 2>&1 || { echo "build failed $v"; continue; }
  timeout 300 python bench.py --steps ${STEPS:-8} --warmup 3 --no-static --no-e2e --no-kernels > gpurun_out/item_ab.log 2>&1
  python - "$v" <<'PY'
import json, sys
for l in open("gpurun_out/item_ab.log"):
    if l.startswith("{"):
        d = json.loads(l)
        x = d["phase_latency"]["XFER"]
        print(sys.argv[1], "value", d["value"], "item_us", x["kl_device_us_mean"], "body_us", x["kl_body_us_mean"],
              "frac", d["roofline"]["frac"])
PY
done
done
python -m paper_conf_sc_senguptagsp14_b200.build >/dev/null 2>&1
