#!/bin/bash
# Build A/B variants of the library into ab/<name>.so (here, no GPU needed):
#   scripts/build_ab.sh name1 "flags1" name2 "flags2" ...
set -eu
mkdir -p ab
while [ $# -ge 2 ]; do
  name=$1; flags=$2; shift 2
  NBODY_NVCC_FLAGS="$flags" python - "$name" <<'PY'
import os, sys
from paper_conf_sc_casselldahg24_b200 import build as B
B.LIB = os.path.abspath(f"ab/{sys.argv[1]}.so")
B.build(force=True)
print(B.LIB, os.environ.get("NBODY_NVCC_FLAGS", ""))
PY
done
