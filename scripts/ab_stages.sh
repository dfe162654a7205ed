#!/bin/bash
# A/B timing of all stages on the GPU box: scripts/ab_stages.sh "<flags A>" "<flags B>" ...
# Each flag set rebuilds the library (NBODY_NVCC_FLAGS) and prints the stage
# times of the 3rd force pass at disks 1e7.
set -u
for flags in "$@"; do
  NBODY_NVCC_FLAGS="$flags" python -m paper_conf_sc_casselldahg24_b200.build --force > /dev/null 2>&1 || { echo "build failed: $flags"; continue; }
  echo "== flags: '$flags'"
  timeout 300 python scripts/run_pass.py --passes 3 | tail -1
done
python -m paper_conf_sc_casselldahg24_b200.build --force > /dev/null 2>&1
