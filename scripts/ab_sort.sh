#!/bin/bash
# A/B of sort tile shapes: libraries prebuilt as ab/sort_<threads>x<items>.so
# (scripts/ab_libs-style; prints ms_sort of 3 passes at disks 1e7 and plummer 1e6)
set -u
for rep in 1 2; do
  for lib in "$@"; do
    a=$(timeout 300 python scripts/run_pass.py --lib $lib --passes 3 | tail -1 | grep -o "'ms_sort': [0-9.]*")
    echo "$rep $lib disks1e7 $a"
  done
done
