#!/bin/bash
# compute-sanitizer over every kernel of the step (GPU box).  Logs to
# gpurun_out/<tag>_sanitizer_<tool>.log; exit status != 0 if any tool reports
# an error.  The second library build (tiny list capacities) drives K6's
# overflow paths under the sanitizer too.
# usage: scripts/sanitize.sh <tag> [n]
set -u
tag=${1:-r02}
n=${2:-30000}
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -m paper_conf_sc_casselldahg24_b200.build > /dev/null
rc=0
for tool in memcheck racecheck synccheck initcheck; do
  log=gpurun_out/${tag}_sanitizer_${tool}.log
  compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 50 python scripts/sanitize_pass.py --n $n > $log 2>&1
  r=$?
  echo "$tool exit=$r" | tee -a $log
  [ $r -ne 0 ] && rc=1
done
# small capacities: spill walks and the box guard on every warp
lib=/tmp/libnbody_smallcaps_san.so
NBODY_NVCC_FLAGS="-DNBODY_CAP_T=64 -DNBODY_CAP_F=32 -DNBODY_CAP_P=32 -DNBODY_CAP_A=64 -DNBODY_QCAP_A=64 -DNBODY_QCAP_P=32 -DNBODY_QCAP_F=32 -DNBODY_QCAP_T=64" \
  python -c "from paper_conf_sc_casselldahg24_b200 import build as B; B.LIB='$lib'; B.build(force=True)"
for tool in memcheck racecheck; do
  log=gpurun_out/${tag}_sanitizer_${tool}_smallcaps.log
  NBODY_TEST_LIB=$lib compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 50 \
    python scripts/sanitize_pass.py --n $n > $log 2>&1
  r=$?
  echo "$tool (small caps) exit=$r" | tee -a $log
  [ $r -ne 0 ] && rc=1
done
exit $rc
