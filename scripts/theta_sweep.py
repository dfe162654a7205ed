"""Config 5: theta sweep 0.3 / 0.5 / 0.8 at N = 1e7, uniform (seed 5) vs
clustered (seed 6), monopole and (NEXT-4) quadrupole.  Reports K6 time, step
time, interactions/body and the Barnes-Hut error against the exact direct sum
(NEXT-1 GPU all-pairs kernel, fp64) on sampled bodies.  Markdown to stdout."""
import argparse
import os
import statistics
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_casselldahg24_b200 import NBody  # noqa: E402
from workloads import generate  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=10_000_000)
ap.add_argument("--samples", type=int, default=1000)
ap.add_argument("--steps", type=int, default=3)
ap.add_argument("--multipoles", default="1,2")
a = ap.parse_args()

print("| workload | theta | multipole | force ms | step ms | interactions/body | err median | err p99 | err max | err rms |")
print("|---|---|---|---|---|---|---|---|---|---|")
for name, seed in (("uniform", 5), ("clustered", 6)):
    pos, vel, mass = generate(name, a.n, seed)
    ids = np.random.default_rng(seed).choice(a.n, a.samples, replace=False)
    exact = None
    for theta in (0.3, 0.5, 0.8):
        for mp in (int(x) for x in a.multipoles.split(",")):
            sim = NBody(a.n, theta, 1e-3, 1e-3, key_bits=16, use_graph=False, multipole=mp)
            sim.set_option(5, 1)
            sim.set_bodies(pos, vel, mass)
            sim.compute_accel()  # the accuracy pass (positions unchanged)
            bh = sim.get_accel()[ids]
            if exact is None:
                exact = sim.direct_accel(ids)
            err = np.linalg.norm(bh - exact, axis=1) / np.linalg.norm(exact, axis=1)
            f, t = [], []
            for _ in range(a.steps):
                sim.step(1)
                s = sim.stats()
                f.append(s["ms_force"])
                t.append(sum(s[k] for k in ("ms_bbox_keys", "ms_sort", "ms_build", "ms_force", "ms_update")))
            inter = sim.stats()["interactions"] / a.n
            print(f"| {name} | {theta} | {'quad' if mp == 2 else 'mono'} | {statistics.mean(f):.2f} | "
                  f"{statistics.mean(t):.2f} | {inter:.0f} | {np.median(err):.2e} | {np.quantile(err, 0.99):.2e} | "
                  f"{err.max():.2e} | {np.sqrt(np.mean(err ** 2)):.2e} |", flush=True)
            sim.close()
