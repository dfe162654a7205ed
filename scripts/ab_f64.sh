#!/bin/bash
# A/B timing of the FP64-mode K6 (NEXT-2) on the GPU box: scripts/ab_f64.sh "<flags A>" ...
set -u
for flags in "$@"; do
  NBODY_NVCC_FLAGS="$flags" python -m paper_conf_sc_casselldahg24_b200.build --force > /dev/null 2>&1 || { echo "build failed: $flags"; continue; }
  echo "== flags: '$flags'"
  timeout 300 python scripts/run_pass.py --passes 2 --precision 64 | tail -1 | grep -o "'ms_force': [0-9.]*"
done
python -m paper_conf_sc_casselldahg24_b200.build --force > /dev/null 2>&1
