"""A/B of the NEXT-1 all-pairs kernel: python scripts/ab_allpairs.py --lib ab/x.so
(disks N = 10^7 sources, 2^17 sampled targets; prints the kernel time and
its FP32-pipe fraction at 20 flop per interaction)."""
import argparse
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--lib", default="")
ap.add_argument("--n", type=int, default=10_000_000)
ap.add_argument("--nt", type=int, default=1 << 17)
a = ap.parse_args()
from paper_conf_sc_casselldahg24_b200 import _capi  # noqa: E402
from paper_conf_sc_casselldahg24_b200 import build as B  # noqa: E402
if a.lib:
    B.LIB = os.path.abspath(a.lib)
    _probe = ctypes.CDLL(B.LIB)
    for _name in list(_capi.SIGNATURES):
        if not hasattr(_probe, _name):
            del _capi.SIGNATURES[_name]
_capi.load(build_if_needed=not a.lib)
from paper_conf_sc_casselldahg24_b200 import NBody  # noqa: E402
from workloads import generate  # noqa: E402

pos, vel, mass = generate("disks", a.n, 3)
sim = NBody(a.n, 0.5, 1e-3, 1e-3, device=0)
sim.set_bodies(pos, vel, mass)
ids = np.sort(np.random.default_rng(11).choice(a.n, a.nt, replace=False))
sim.allpairs_accel(ids[:4096], timed=True)
ms = min(sim.allpairs_accel(ids, timed=True)[1] for _ in range(2))
tf = 20.0 * a.nt * a.n / (ms / 1e3) / 1e12
print(f"{a.lib} allpairs {ms:.2f} ms  {tf:.2f} TFLOP/s  frac {tf / 74.44992:.3f}")
