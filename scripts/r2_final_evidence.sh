#!/bin/bash
# Round-2 final evidence at HEAD (GPU box): tests, smoke, bench, launch list,
# ncu of K6 and the other kernels, config 4 on one GPU, theta sweep, lane use.
set -u
tag=${1:-r02i}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/${tag}_pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/${tag}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.log 2>&1; echo smoke=$?
bash scripts/evidence.sh $tag
timeout 900 python bench.py --config cfg4 --steps 3 --warmup 3 --repeats 1 --no-cpu-baseline --no-extras \
  > gpurun_out/${tag}_bench_cfg4_1gpu.json 2> gpurun_out/${tag}_bench_cfg4_1gpu.err; echo cfg4=$?
timeout 1800 python scripts/theta_sweep.py > gpurun_out/${tag}_theta_sweep.md 2> gpurun_out/${tag}_theta_sweep.err; echo sweep=$?
bash scripts/theta_lane_util.sh; cp gpurun_out/theta_lane_util.jsonl gpurun_out/${tag}_theta_lane_util.jsonl
