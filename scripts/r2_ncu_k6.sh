# one ncu --set full capture of K6 (disks 1e7) with source counters (GPU box)
set -u
mkdir -p gpurun_out
tag=${1:-k6}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_force_grouped -s 1 -c 1 -o gpurun_out/force_${tag} \
  python scripts/run_pass.py --passes 2 > gpurun_out/ncu_${tag}.log 2>&1; echo ncu=$?
