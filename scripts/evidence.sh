#!/bin/bash
# Bench + ncu evidence for profiles/ (run on the GPU box).  Usage: scripts/evidence.sh <tag>
set -u
tag=${1:-r01}
mkdir -p gpurun_out
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_${tag}.json 2> gpurun_out/bench_${tag}.err; echo bench=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_${tag}.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-extras > /dev/null 2>&1; echo launches=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_force_grouped -s 1 -c 1 -o gpurun_out/force_${tag} \
  python scripts/run_pass.py --passes 2 > /dev/null 2>&1; echo ncu_force=$?
timeout 900 ncu --set full --clock-control none -k regex:"k_onesweep|k_build|k_permute|k_keys|k_bbox|k_leapfrog" -s 13 -c 13 -o gpurun_out/build_${tag} \
  python scripts/run_pass.py --passes 3 > /dev/null 2>&1; echo ncu_build=$?
