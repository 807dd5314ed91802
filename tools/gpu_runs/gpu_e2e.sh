#!/bin/bash
cd $GRAFT_REPO_ROOT
for ct in 6 12; do
  STRINGS_COPY_THREADS=$ct timeout 300 python bench.py --no-static --no-kernels > gpurun_out/e2e_$ct.log 2>/dev/null
  echo "threads $ct"; python tools/show_bench.py gpurun_out/e2e_$ct.log value e2e e2e_pinned
done
