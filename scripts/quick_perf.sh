#!/bin/bash
# quick correctness + timing sweep used during kernel iteration (on the GPU box)
set -u
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
for v in 0 1; do
  timeout 300 python scripts/run_pass.py --passes 3 --traversal $v 2>&1 | tail -1
  timeout 300 python scripts/run_pass.py --workload plummer --n 1000000 --seed 2 --passes 2 --traversal $v | tail -1
done
