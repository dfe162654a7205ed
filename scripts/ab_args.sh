#!/bin/bash
# A/B of prebuilt libraries with extra run_pass.py arguments:
# scripts/ab_args.sh "<run_pass args>" lib1.so lib2.so ...   (K6 time, 3 passes, twice)
set -u
args=$1; shift
for rep in 1 2; do
  for lib in "$@"; do
    a=$(timeout 600 python scripts/run_pass.py --lib $lib --passes 3 $args | tail -1 | grep -o "'ms_force': [0-9.]*")
    echo "$rep $lib [$args] $a"
  done
done
