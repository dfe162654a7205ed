"""Per-phase SM cycles of the onesweep tiles (design build with
-DNBODY_SORT_PROFILE): python scripts/sort_profile.py --lib ab/sortprof.so"""
import argparse
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
ap = argparse.ArgumentParser()
ap.add_argument("--lib", required=True)
a = ap.parse_args()
from paper_conf_sc_casselldahg24_b200 import _capi  # noqa: E402
from paper_conf_sc_casselldahg24_b200 import build as B  # noqa: E402
B.LIB = os.path.abspath(a.lib)
_capi.load(build_if_needed=False)
from paper_conf_sc_casselldahg24_b200 import NBody  # noqa: E402
from workloads import generate  # noqa: E402

lib = ctypes.CDLL(B.LIB)
buf = (ctypes.c_uint64 * 6)()
n = 10_000_000
pos, vel, mass = generate("disks", n, 3)
sim = NBody(n, 0.5, 1e-3, 1e-3, use_graph=False, device=0)
sim.set_bodies(pos, vel, mass)
sim.step(1)
sim.sync()
lib.nbody_debug_sort_profile(buf)
sim.step(1)
sim.sync()
lib.nbody_debug_sort_profile(buf)
v = list(buf)
tiles = v[5]
names = ["tile id + zero", "loads + warp ranking", "prefixes + publish", "smem scatter + look-back", "global scatter"]
tot = sum(v[:5])
print(f"tiles {tiles} (6 passes); mean SM cycles per tile {tot / tiles:.0f}")
for nm, x in zip(names, v[:5]):
    print(f"  {nm:28s} {x / tiles:8.0f} cycles  {100 * x / tot:5.1f} %")
