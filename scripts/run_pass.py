"""Run a few force passes of the CUDA path (graphs off) for ncu captures.

python scripts/run_pass.py [--workload disks] [--n 10000000] [--passes 2] [--traversal 0]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="disks")
ap.add_argument("--n", type=int, default=10_000_000)
ap.add_argument("--seed", type=int, default=3)
ap.add_argument("--theta", type=float, default=0.5)
ap.add_argument("--passes", type=int, default=2)
ap.add_argument("--traversal", type=int, default=0)
ap.add_argument("--key-bits", type=int, default=16)
ap.add_argument("--multipole", type=int, default=1)
ap.add_argument("--precision", type=int, default=32)
ap.add_argument("--lib", default="", help="load this libnbody_b200.so instead of the in-tree build (A/B runs)")
a = ap.parse_args()
if a.lib:  # an older build may lack later entry points: bind only what it exports
    import ctypes
    from paper_conf_sc_casselldahg24_b200 import _capi
    from paper_conf_sc_casselldahg24_b200 import build as B
    B.LIB = os.path.abspath(a.lib)
    _probe = ctypes.CDLL(B.LIB)
    for _name in list(_capi.SIGNATURES):
        if not hasattr(_probe, _name):
            del _capi.SIGNATURES[_name]
    _capi.load(build_if_needed=False)  # never rebuild the A/B library from the current sources
from paper_conf_sc_casselldahg24_b200 import NBody  # noqa: E402
from workloads import generate  # noqa: E402

pos, vel, mass = generate(a.workload, a.n, a.seed)
sim = NBody(a.n, a.theta, 1e-3, 1e-3, key_bits=a.key_bits, use_graph=False, traversal=a.traversal,
            multipole=a.multipole, precision=a.precision)
sim.set_option(5, 1)
sim.set_bodies(pos, vel, mass)
for _ in range(a.passes):
    sim.step(1)
    s = sim.stats()
    print({k: s[k] for k in ("interactions", "ms_bbox_keys", "ms_sort", "ms_build", "ms_force", "ms_update")},
          flush=True)
