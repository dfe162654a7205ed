"""Driver for compute-sanitizer (VERDICT r1 missing #5).

Runs every kernel of the step once at small N with graphs off, so the
sanitizer sees plain launches: one force pass + one step for the default
traversal, the mask walk, the paper's skip-list walk, quadrupoles, tree
reuse, the FP64 mode, the fused peer exchange with 2 contexts (balanced
ranges) and the small-capacity overflow paths when the library was built
with them.  No torch import (device 0 is selected through the C ABI).
python scripts/sanitize_pass.py [--n 30000]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from paper_conf_sc_casselldahg24_b200 import build as B  # noqa: E402

if os.environ.get("NBODY_TEST_LIB"):  # a design build (e.g. tiny list capacities) in place of the product
    B.LIB = os.environ["NBODY_TEST_LIB"]
from paper_conf_sc_casselldahg24_b200 import NBody  # noqa: E402
from workloads import generate  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=30_000)
a = ap.parse_args()
n = a.n
pos, vel, mass = generate("disks", n, 3)


def run(tag, **kw):
    s = NBody(n, 0.5, 1e-3, 1e-3, use_graph=False, device=0, **kw)
    if kw.get("precision") == 64:
        s.set_bodies(pos.astype(np.float64), vel.astype(np.float64), mass.astype(np.float64))
    else:
        s.set_bodies(pos, vel, mass)
    s.compute_accel()
    s.step(2)
    s.sync()
    acc = s.get_accel64() if kw.get("precision") == 64 else s.get_accel()
    assert np.isfinite(acc).all()
    print(f"{tag}: ok, {int(s.get_interactions().sum())} interactions", flush=True)
    s.close()


run("variant0")
run("variant1 mask walk", traversal=1)
run("variant2 skip list", traversal=2)
run("quadrupoles", multipole=2)
run("fp64 mode", precision=64)
s = NBody(n, 0.5, 1e-3, 1e-3, use_graph=False, device=0)
s.set_option(7, 2)  # tree reuse
s.set_bodies(pos, vel, mass)
s.step(3)
s.sync()
print("tree reuse: ok", flush=True)
s.close()
# the sanitizer serialises kernels, so ranks on one GPU whose device barriers
# wait for each other would deadlock: one rank exercises the exchange kernels
# (scatter stores, barriers, partition) against itself
ranks = [NBody(n, 0.5, 1e-3, 1e-3, use_graph=False, device=0, balance=True) for _ in range(1)]
NBody.attach_peers_local(ranks)
for r in ranks:
    r.set_bodies(pos, vel, mass)
for _ in range(2):
    for r in ranks:
        r.step(1)
for r in ranks:
    r.sync()
print("peer exchange kernels, one rank (balanced): ok", flush=True)
for r in ranks:
    r.close()
ids = np.arange(0, n, 97)
s = NBody(n, 0.5, 1e-3, 1e-3, use_graph=False, device=0)
s.set_bodies(pos, vel, mass)
assert np.isfinite(s.direct_accel(ids)).all()
print("all-pairs: ok", flush=True)
