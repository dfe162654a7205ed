"""Work balance of the Hilbert-range partition: interactions per
rank for equal-count slices vs cost-weighted slices, from one force pass."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_casselldahg24_b200 import NBody  # noqa: E402
from workloads import CONFIGS, generate  # noqa: E402

for cfg_name in ("cfg3", "cfg2"):
    cfg = CONFIGS[cfg_name]
    n = cfg["n"]
    pos, vel, mass = generate(cfg["workload"], n, cfg["seed"])
    sim = NBody(n, cfg["theta"], cfg["eps"], cfg["dt"])
    sim.set_bodies(pos, vel, mass)
    sim.compute_accel()
    ids = sim.get_state()[1][:, 3].view(np.int32)
    cost = sim.get_interactions()[ids].astype(np.float64)  # slot order
    for g in (2, 4, 8):
        s = -(-n // g)
        s = -(-s // 32) * 32
        eq = [cost[r * s:min(n, (r + 1) * s)].sum() for r in range(g)]
        cum = np.cumsum(cost)
        cuts = [0] + [int(np.searchsorted(cum, cum[-1] * r / g)) // 32 * 32 for r in range(1, g)] + [n]
        cw = [cost[cuts[r]:cuts[r + 1]].sum() for r in range(g)]
        print(f"{cfg_name} G={g}: equal-count max/mean {max(eq) / np.mean(eq):.3f}; "
              f"cost-weighted max/mean {max(cw) / np.mean(cw):.3f}", flush=True)
