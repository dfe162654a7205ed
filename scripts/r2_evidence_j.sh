#!/bin/bash
# Evidence refresh at HEAD (GPU box): bench + launch list + ncu (scripts/evidence.sh),
# smoke, config 4 on one GPU.
set -u
tag=${1:-r02j}
bash scripts/evidence.sh $tag
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.log 2>&1; echo smoke=$?
timeout 900 python bench.py --config cfg4 --steps 3 --warmup 3 --repeats 1 --no-cpu-baseline --no-extras \
  > gpurun_out/${tag}_bench_cfg4_1gpu.json 2> gpurun_out/${tag}_bench_cfg4_1gpu.err; echo cfg4=$?
