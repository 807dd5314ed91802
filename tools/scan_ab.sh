#!/bin/bash
# SCAN variants on the box: two-pass vs waves of several sizes (2^28 u32, 148 CTAs),
# then ncu DRAM bytes / L2 hit rate of one launch of the default build.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for v in ${SCAN_AB_VARIANTS:-"-DSTRINGS_SCAN_TWOPASS=1" "-DSTRINGS_SCAN_WAVE_MB=6" "-DSTRINGS_SCAN_WAVE_MB=10" "-DSTRINGS_SCAN_WAVE_MB=14" "-DSTRINGS_SCAN_WAVE_MB=20"}; do
  STRINGS_NVCC_EXTRA="${v//,/ }" python -m paper_conf_sc_senguptagsp14_b200.build >/dev/null 2>&1 || { echo "build failed $v"; continue; }
  echo "== $v"; timeout 120 python tools/scan_probe.py ${SCAN_AB_PROBE:---quick}
  timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct \
     -k regex:oneshot_kernel --launch-skip 1 -c 1 --clock-control none python tools/scan_probe.py --quick --once 2>&1 \
     | grep -E "gpu__time|dram__bytes|lts__t_sector" 
done
python -m paper_conf_sc_senguptagsp14_b200.build >/dev/null 2>&1
