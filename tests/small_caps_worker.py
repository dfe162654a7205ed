"""Subprocess body of test_small_caps_gpu.py: loads a K6 build with tiny list
capacities (path in NBODY_TEST_LIB) in place of the product library, runs
force passes against the oracle and prints one JSON line.  Not a test module
(no test_ prefix); only tests/test_small_caps_gpu.py runs it."""
import ctypes as C
import json
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(HERE))
sys.path.insert(0, HERE)

import numpy as np  # noqa: E402

from paper_conf_sc_casselldahg24_b200 import build as B  # noqa: E402

B.LIB = os.environ["NBODY_TEST_LIB"]
from oracle import oracle as O  # noqa: E402
from paper_conf_sc_casselldahg24_b200 import NBody, _capi  # noqa: E402
from parity_utils import rel_errors  # noqa: E402
from workloads import generate  # noqa: E402

lib = _capi.load(build_if_needed=False)
out = []
for name, n, seed, theta, quad in [("disks", 40_000, 3, 0.5, False), ("clustered", 30_001, 4, 0.8, False),
                                   ("plummer", 20_000, 5, 0.3, False), ("plummer", 20_000, 6, 0.5, True)]:
    pos, vel, mass = generate(name, n, seed)
    buf = (C.c_uint64 * 52)()
    lib.nbody_debug_force_stats(buf, 52)  # reset the counters
    sim = NBody(n, theta, 1e-3, 1e-3, key_bits=16, use_graph=False, multipole=2 if quad else 1)
    sim.set_bodies(pos, vel, mass)
    sim.compute_accel()
    sim.sync()
    lane_util = sim.stats()["lane_util"]  # peeks at the counters (no reset)
    got = lib.nbody_debug_force_stats(buf, 52)
    ref = O.step(pos, vel, mass, theta=theta, eps=1e-3, dt=1e-3, key_bits=16, integrate=False, quad=quad)
    cnt = sim.get_interactions()[ref.ids]
    e = rel_errors(sim.get_accel()[ref.ids], ref.acc)
    out.append({"case": f"{name} n={n} theta={theta} quad={quad}", "stats_len": got,
                "spill_walks": int(buf[14]), "guard_handovers": int(buf[36]), "no_sg_lists": int(buf[49]),
                "counts_equal": bool((cnt == ref.count).all()), "lane_util": lane_util,
                "rms": float(np.sqrt(np.mean(e ** 2))), "max": float(e.max())})
    sim.close()
print(json.dumps(out))
