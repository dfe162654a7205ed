"""Projected multi-GPU step times from ONE GPU (no multi-GPU box here).

G contexts with equal Hilbert ranges [A21] (nbody_set_partition) on the one
GPU; each rank's force pass is timed alone (graphs off, CUDA events), after
two warm-up steps whose owned slices are exchanged with nbody_copy_owned.
Projected step(G) = replicated S1-S5 (the same on every rank) + max over
ranks of (K6a + K6) + max over ranks of K7 + the all-gather's bytes over
NVLink 5 ((G-1)/G x N x 32 B at 800 GB/s).  With cost-weighted ranges the
K6 term approaches the mean over ranks, also reported.
python scripts/scale_projection.py [--n 10000000]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sc_casselldahg24_b200 import NBody  # noqa: E402
from workloads import generate  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=10_000_000)
ap.add_argument("--workload", default="disks")
ap.add_argument("--seed", type=int, default=3)
a = ap.parse_args()
n = a.n
pos, vel, mass = generate(a.workload, n, a.seed)
print(f"| G | replicated S1-S5 ms | K6 max ms | K6 mean ms | K7 max ms | exchange ms (est.) | projected step ms | "
      f"speed-up | with balanced K6 | speed-up |")
print("|---|---|---|---|---|---|---|---|---|---|")
base = None
for G in (1, 2, 4, 8):
    ranks = [NBody(n, 0.5, 1e-3, 1e-3, use_graph=False) for _ in range(G)]
    for r, s in enumerate(ranks):
        if G > 1:
            s.set_partition(r, G)
        s.set_option(5, 1)  # NBODY_OPT_TIMING
        s.set_bodies(pos, vel, mass)
    stats = []
    for it in range(3):
        stats = []
        for s in ranks:
            s.step(1)
            s.sync()
            stats.append(s.stats())
        for dst in ranks:
            for src in ranks:
                if src is not dst:
                    dst.copy_owned_from(src)
    rep = float(np.median([st["ms_bbox_keys"] + st["ms_sort"] + st["ms_build"] for st in stats]))
    k6 = [st["ms_force"] for st in stats]
    k7 = max(st["ms_update"] for st in stats)
    xch = (G - 1) / G * n * 32 / 800e9 * 1e3 if G > 1 else 0.0
    step = rep + max(k6) + k7 + xch
    bal = rep + float(np.mean(k6)) + k7 + xch
    if base is None:
        base = step
    print(f"| {G} | {rep:.2f} | {max(k6):.2f} | {np.mean(k6):.2f} | {k7:.3f} | {xch:.3f} | {step:.2f} | "
          f"{base / step:.2f} | {bal:.2f} | {base / bal:.2f} |", flush=True)
    for s in ranks:
        s.close()
