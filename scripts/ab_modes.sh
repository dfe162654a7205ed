#!/bin/bash
# A/B of prebuilt libraries in the FP64 and quadrupole modes (K6 ms, disks 10^7, GPU box)
set -u
for rep in 1 2; do
  for lib in "$@"; do
    a=$(timeout 300 python scripts/run_pass.py --lib $lib --precision 64 --passes 2 | tail -1 | grep -o "'ms_force': [0-9.]*")
    b=$(timeout 300 python scripts/run_pass.py --lib $lib --multipole 2 --passes 2 | tail -1 | grep -o "'ms_force': [0-9.]*")
    echo "$rep $lib fp64 $a quad $b"
  done
done
