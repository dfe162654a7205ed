#!/bin/bash
# rebuild with different K6 list capacities / occupancy targets and time K6 (GPU box)
for cfg in "352 8 96 64" "192 8 128 128" "256 7 160 128" "160 8 160 96" "512 5 192 160"; do
  set -- $cfg
  NBODY_NVCC_FLAGS="-DNBODY_CAP_T=$1 -DNBODY_V0_MINB=$2 -DNBODY_CAP_F=$3 -DNBODY_CAP_P=$4" python -m paper_conf_sc_casselldahg24_b200.build --force > /dev/null 2>&1
  echo "CAP_T=$1 MINB=$2 F=$3 P=$4"
  timeout 300 python scripts/run_pass.py --passes 2 | tail -1 | grep -o "'ms_force': [0-9.]*"
  timeout 300 python scripts/run_pass.py --workload plummer --n 1000000 --seed 2 --passes 2 | tail -1 | grep -o "'ms_force': [0-9.]*"
done
