#!/bin/bash
# A/B of prebuilt libraries on the theta-sweep workloads (K6 + K6a ms, GPU box)
set -u
for lib in "$@"; do
  for w in "uniform 5 0.3" "clustered 6 0.3" "clustered 6 0.5" "uniform 5 0.8"; do
    set -- $w
    a=$(timeout 300 python scripts/run_pass.py --lib $lib --workload $1 --seed $2 --theta $3 --passes 2 | tail -1 | grep -o "'ms_force': [0-9.]*")
    echo "$lib $1 $3 $a"
  done
done
