#!/bin/bash
# A/B timing of K6 variants on the GPU box: scripts/ab_force.sh "<flags A>" "<flags B>" ...
# Each flag set rebuilds the library (NBODY_NVCC_FLAGS) and times 3 force passes
# at disks 1e7 and plummer 1e6.
set -u
for flags in "$@"; do
  NBODY_NVCC_FLAGS="$flags" python -m paper_conf_sc_casselldahg24_b200.build --force > /dev/null 2>&1 || { echo "build failed: $flags"; continue; }
  echo "== flags: '$flags'"
  timeout 300 python scripts/run_pass.py --passes 3 | tail -1 | grep -o "'ms_force': [0-9.]*"
  timeout 300 python scripts/run_pass.py --workload plummer --n 1000000 --seed 2 --passes 3 | tail -1 | grep -o "'ms_force': [0-9.]*"
done
python -m paper_conf_sc_casselldahg24_b200.build --force > /dev/null 2>&1
