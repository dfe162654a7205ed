#!/bin/bash
# Config 5 lane utilisation (GPU box): K6 design counters for the theta sweep's
# monopole runs (uniform seed 5 / clustered seed 6, N = 1e7, theta 0.3/0.5/0.8)
set -u
out=gpurun_out/theta_lane_util.jsonl
rm -f $out
first=1
for w in "uniform 5" "clustered 6"; do
  set -- $w
  for th in 0.3 0.5 0.8; do
    nb=$([ $first = 1 ] && echo "" || echo "--no-build")
    timeout 600 python scripts/k6_stats.py --workload $1 --seed $2 --n 10000000 --theta $th $nb --json $out > /dev/null 2>&1
    echo "$1 $th rc=$?"
    first=0
  done
done
