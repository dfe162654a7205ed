set -u
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo bench=$?; tail -c 3000 gpurun_out/bench.log
timeout 600 python scripts/k6_stats.py > gpurun_out/k6stats_disks.log 2>&1; echo stats=$?
cat gpurun_out/k6stats_disks.log | tail -60
