#!/bin/bash
# The bench's N > 1 path run end to end with every rank on the one GPU of the
# box (validation only, never a performance number): torchrun, peer attach
# over CUDA IPC, cost-weighted ranges, graphs, max-over-ranks timing, e2e.
set -u
for g in 2 4; do
  echo "## G = $g"
  NBODY_BENCH_ONE_DEVICE=1 timeout 600 python -m torch.distributed.run --nproc-per-node $g --master-addr 127.0.0.1 \
    --master-port $((29500 + g)) bench.py --gpus $g --steps 3 --warmup 3 --config cfg2 --no-cpu-baseline --repeats 1 2>&1 | grep '^{' 
done
