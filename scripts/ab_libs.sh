#!/bin/bash
# A/B of prebuilt libraries on one box: scripts/ab_libs.sh lib1.so lib2.so ...
# (K6 time of 3 force passes at disks 1e7 and plummer 1e6, twice, interleaved)
set -u
for rep in 1 2; do
  for lib in "$@"; do
    a=$(timeout 300 python scripts/run_pass.py --lib $lib --passes 3 | tail -1 | grep -o "'ms_force': [0-9.]*")
    b=$(timeout 300 python scripts/run_pass.py --lib $lib --workload plummer --n 1000000 --seed 2 --passes 3 | tail -1 | grep -o "'ms_force': [0-9.]*")
    echo "$rep $lib disks1e7 $a plummer1e6 $b"
  done
done
