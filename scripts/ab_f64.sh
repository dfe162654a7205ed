#!/bin/bash
# A/B of prebuilt libraries in the FP64 mode (K6 time, disks 10^7, 3 passes, twice)
set -u
for rep in 1 2; do
  for lib in "$@"; do
    a=$(timeout 300 python scripts/run_pass.py --lib $lib --precision 64 --passes 3 | tail -1 | grep -o "'ms_force': [0-9.]*")
    echo "$rep $lib fp64 disks1e7 $a"
  done
done
