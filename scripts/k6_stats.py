"""K6 traversal event counts (design instrumentation, GPU box).

Builds a separate library with -DNBODY_K6_STATS into /tmp, loads it in place of
the product library, runs one force pass and prints per-warp averages.
python scripts/k6_stats.py [--workload disks] [--n 10000000] [--seed 3] [--theta 0.5]
"""
import argparse
import ctypes as C
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

kStatNames = ["warps", "A batches", "A nodes", "T batches", "T nodes", "full entries", "partial entries",
              "partial lanes", "full lanes", "fp64 fallbacks", "dense_full calls", "dense_full pairs",
              "dense_part calls", "dense_part pairs", "spill walks", "T batches < 32",
              "T nodes 1-quarter", "T nodes 1-half", "T mask lanes", "partial q-incid", "partial 1-quarter",
              "partial h-incid", "part sum max q", "part sum max h", "T accept lanes", "T open lanes",
              "part max 8grp", "part max 16grp", "part max lane", "T leaf nodes", "T level-1 nodes", "T internal uniform",
              "partial popc 1", "partial popc 2", "partial popc <=4", "partial popc <=8", "A guard handovers", "Q-local max-quarter", "H-local max-half", "general partial", "A nodes decided by 128-box", "A nodes decided by 256-box", "A nodes accepted by 128-box", "A internal nodes", "A internal accepted (warp)", "A expanded (warp)", "T internal decided by quarter-union box", "T internal nodes", "T batches all decided", "warps without super-group lists", "T internal full-mask", "T internal full-mask all-open"]

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="disks")
ap.add_argument("--n", type=int, default=10_000_000)
ap.add_argument("--seed", type=int, default=3)
ap.add_argument("--theta", type=float, default=0.5)
ap.add_argument("--flags", default="")
ap.add_argument("--no-build", action="store_true", help="reuse the stats library built by an earlier run")
ap.add_argument("--json", default="", help="append one JSON record of the per-warp counters to this file")
a = ap.parse_args()

from paper_conf_sc_casselldahg24_b200 import build as B  # noqa: E402

lib = "/tmp/libnbody_b200_stats.so"
os.environ["NBODY_NVCC_FLAGS"] = ("-DNBODY_K6_STATS " + a.flags).strip()
B.LIB = lib
if not (a.no_build and os.path.exists(lib)):
    B.build(force=True)
from paper_conf_sc_casselldahg24_b200 import _capi, NBody  # noqa: E402
from workloads import generate  # noqa: E402

L = _capi.load(build_if_needed=False)
pos, vel, mass = generate(a.workload, a.n, a.seed)
sim = NBody(a.n, a.theta, 1e-3, 1e-3, key_bits=16, use_graph=False)
sim.set_bodies(pos, vel, mass)
buf = (C.c_uint64 * 52)()
L.nbody_debug_force_stats(buf, 52)
sim.compute_accel()
sim.sync()
got = L.nbody_debug_force_stats(buf, 52)
assert got == 52, "library not built with NBODY_K6_STATS"
v = list(buf)
inter = int(sim.get_interactions().sum())
w = v[0]
print(f"{a.workload} N={a.n} theta={a.theta}: interactions {inter} ({inter / a.n:.1f}/body), warps {w}")
for name, x in zip(kStatNames, v):
    print(f"  {name:18s} {x:16d}  per warp {x / w:10.1f}")
pl = v[7] / max(v[6], 1)
print(f"  partial-entry lane use {pl:.2f}/32; full lanes share of interactions {v[8] / inter:.3f}; "
      f"partial lanes share {v[7] / inter:.3f}")
print(f"  T nodes per batch {v[4] / max(v[3], 1):.1f}; A nodes per batch {v[2] / max(v[1], 1):.1f}")

if a.json:
    import json
    rec = {"workload": a.workload, "n": a.n, "seed": a.seed, "theta": a.theta, "interactions": inter,
           "warps": w, "per_warp": {name: x / w for name, x in zip(kStatNames, v)},
           "partial_lane_use": pl, "dense_lane_util": (v[7] + v[8]) / max(32.0 * (v[5] + v[6]), 1.0)}
    with open(a.json, "a") as f:
        f.write(json.dumps(rec) + "\n")
