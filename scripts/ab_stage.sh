#!/bin/bash
# A/B of one stage time of prebuilt libraries: scripts/ab_stage.sh <stage key> lib1.so ...
# (e.g. ms_bbox_keys, ms_sort, ms_build, ms_update; disks 10^7, 3 passes, twice)
set -u
key=$1; shift
for rep in 1 2; do
  for lib in "$@"; do
    a=$(timeout 300 python scripts/run_pass.py --lib $lib --passes 3 | tail -1 | grep -o "'$key': [0-9.]*")
    echo "$rep $lib $a"
  done
done
