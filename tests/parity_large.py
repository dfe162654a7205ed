"""Sampled parity at a large configuration (default: config 4, clustered
Plummer N = 1e8) on one GPU: Hilbert keys and the sort permutation in full,
node records on sampled nodes of every level, forces and interaction counts
on sampled targets, all against the fp64 oracle."""
import argparse
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from oracle import oracle as O  # noqa: E402
from paper_conf_sc_casselldahg24_b200 import NBody  # noqa: E402
from workloads import CONFIGS, generate  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="cfg4")
ap.add_argument("--samples", type=int, default=400)
a = ap.parse_args()
cfg = CONFIGS[a.config]
n = cfg["n"]
t0 = time.time()
pos, vel, mass = generate(cfg["workload"], n, cfg["seed"])
print(f"generate {time.time() - t0:.1f}s", flush=True)
t0 = time.time()
sim = NBody(n, cfg["theta"], cfg["eps"], cfg["dt"], key_bits=16, use_graph=False)
sim.set_option(5, 1)
sim.set_bodies(pos, vel, mass)
sim.compute_accel()
sim.sync()
st = sim.stats()
print(f"gpu pass {time.time() - t0:.1f}s  stage ms: force {st['ms_force']:.1f} sort {st['ms_sort']:.2f} "
      f"build {st['ms_build']:.2f} keys {st['ms_bbox_keys']:.2f}; interactions/body {st['interactions'] / n:.0f}",
      flush=True)
rng = np.random.default_rng(cfg["seed"])
targets = np.sort(rng.choice(n, a.samples, replace=False))
t0 = time.time()
ref = O.step(pos, vel, mass, theta=cfg["theta"], eps=cfg["eps"], dt=cfg["dt"], key_bits=16, integrate=False,
             targets=targets)
print(f"oracle {time.time() - t0:.1f}s", flush=True)
ok = True
kg = sim.debug_keys()
ok &= bool((kg == ref.keys).all())
print("keys bit-exact:", ok, flush=True)
pg = sim.debug_perm()
pk = bool((pg == ref.perm).all())
ok &= pk
print("perm bit-exact:", pk, flush=True)
del kg, pg
bad_levels = 0
for l in range(1, ref.tree.L + 1):
    pred, rec, box = sim.debug_level(l)
    d = ref.tree.level(l)
    sel = slice(None) if len(pred) <= 4096 else rng.choice(len(pred), 4096, replace=False)
    good = (pred[sel, :3] == d.com[sel]).all() and (pred[sel, 3] == d.s2[sel]).all() and \
        (rec[sel, :3] == d.c32[sel]).all() and (rec[sel, 3] == d.m32[sel]).all() and \
        (box[sel, :3] == d.lo[sel]).all() and (box[sel, 3:] == d.hi[sel]).all()
    bad_levels += not good
print("node records bit-exact on sampled nodes of all", ref.tree.L, "levels:", bad_levels == 0, flush=True)
ok &= bad_levels == 0
acc = sim.get_accel()[ref.ids[targets]]
cnt = sim.get_interactions()[ref.ids[targets]]
ce = bool((cnt == ref.count).all())
e = np.linalg.norm(acc - ref.acc, axis=1) / np.linalg.norm(ref.acc, axis=1)
rms, mx = float(np.sqrt(np.mean(e ** 2))), float(e.max())
print(f"counts equal: {ce}; acc rel err rms {rms:.2e} max {mx:.2e} ({a.samples} targets)", flush=True)
ok &= ce and rms <= 1e-4 and mx <= 1e-2
print("PARITY", "OK" if ok else "FAILED")
sys.exit(0 if ok else 1)
