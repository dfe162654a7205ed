"""CPU pin of K2's table-driven Hilbert automaton (no GPU needed).

The CUDA path evaluates Skilling's transform [17] as a 48-state
automaton whose tables are generated at compile time (k_bbox_keys.cu).  This
test compiles that file's table generator and `hilbert_key` for the host
with nvcc and compares them with the oracle's Skilling routine on random
cells for every b in [1, 21] plus the curve ends; the GPU parity tests check
the same on the device."""
import os
import random
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "paper_conf_sc_casselldahg24_b200", "csrc", "k_bbox_keys.cu")

HARNESS = r'''
#include "%s"
#include <cstdio>
int main() {
  unsigned x, y, z; int b;
  std::printf("%%d\n", nb::kHilbertFsm.nstates);
  while (std::scanf("%%u %%u %%u %%d", &x, &y, &z, &b) == 4)
    std::printf("%%llu\n", nb::hilbert_key<unsigned long long>(x, y, z, b, nb::kHilbertFsm.t2, nb::kHilbertFsm.t1));
  return 0;
}
'''


@pytest.fixture(scope="module")
def fsm_exe(tmp_path_factory):
    nvcc = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
    if not os.path.exists(nvcc):
        pytest.skip("nvcc not available")
    d = tmp_path_factory.mktemp("fsm")
    cu = d / "h.cu"
    cu.write_text(HARNESS % SRC)
    exe = d / "h"
    subprocess.run([nvcc, "-std=c++17", "-O1", "-gencode", "arch=compute_100a,code=sm_100a", "-I",
                    os.path.join(ROOT, "include"), "-o", str(exe), str(cu)], check=True, capture_output=True)
    return str(exe)


def test_fsm_keys_equal_oracle_skilling(fsm_exe, oracle):
    rng = random.Random(7)
    cases = []
    for b in range(1, 22):
        m = (1 << b) - 1
        cases += [(0, 0, 0, b), (m, 0, 0, b), (0, 0, m, b), (m, m, m, b)]
        cases += [(rng.randint(0, m), rng.randint(0, m), rng.randint(0, m), b) for _ in range(300)]
    inp = "\n".join(f"{x} {y} {z} {b}" for x, y, z, b in cases) + "\n"
    out = subprocess.run([fsm_exe], input=inp, capture_output=True, text=True, check=True).stdout.split()
    assert int(out[0]) == 48, "Skilling's 3-D transform has 48 (transform, parity) states"
    got = [int(v) for v in out[1:]]
    want = [oracle.hilbert_index(x, y, z, b) for x, y, z, b in cases]
    assert got == want
