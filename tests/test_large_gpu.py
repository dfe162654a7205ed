"""Config 4 (clustered Plummer, N = 1e8) sampled parity on one GPU: keys and
the permutation in full, node records on sampled nodes of all 27 levels,
forces and counts on sampled targets (tests/parity_large.py; ~90 s)."""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.gpu
@pytest.mark.slow
def test_config4_100M_sampled_parity():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tests", "parity_large.py"), "--config", "cfg4",
                        "--samples", "300"], capture_output=True, text=True, timeout=1200)
    assert r.returncode == 0 and "PARITY OK" in r.stdout, r.stdout[-3000:] + r.stderr[-3000:]
