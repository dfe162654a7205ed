#!/bin/bash
set -u
for flags in "$@"; do
  NBODY_NVCC_FLAGS="$flags" python -m paper_conf_sc_casselldahg24_b200.build --force > /dev/null 2>&1 || { echo "build failed: $flags"; continue; }
  echo "== flags: '$flags'"
  timeout 300 python scripts/run_pass.py --passes 2 --multipole 2 --workload uniform --seed 5 | tail -1 | grep -o "'ms_force': [0-9.]*"
done
python -m paper_conf_sc_casselldahg24_b200.build --force > /dev/null 2>&1
