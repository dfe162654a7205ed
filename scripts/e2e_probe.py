"""Attribute the end-to-end overhead per step (GPU box): the bench's pipelined
host calls with parts switched off.  python scripts/e2e_probe.py [--steps 20]"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_casselldahg24_b200 import NBody  # noqa: E402
from workloads import generate  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=20)
ap.add_argument("--n", type=int, default=10_000_000)
a = ap.parse_args()
pos, vel, mass = generate("disks", a.n, 3)
stream = torch.cuda.Stream()
sim = NBody(a.n, 0.5, 1e-3, 1e-3, key_bits=16, stream=stream.cuda_stream)
sim.set_bodies(pos, vel, mass)
hp, hv, hm = (torch.from_numpy(x).pin_memory() for x in (pos, vel, mass))
outs = [torch.empty((a.n, 3), dtype=torch.float32).pin_memory() for _ in range(2)]


def run(label, up, down):
    def one(k):
        if up:
            sim.set_bodies_async(hp, hv, hm)
        sim.step(1)
        if down:
            sim.get_positions_async(outs[k & 1])
    for k in range(3):
        one(k)
    sim.sync()
    t0 = time.perf_counter()
    for k in range(a.steps):
        one(k)
    sim.sync()
    ms = 1e3 * (time.perf_counter() - t0) / a.steps
    print(f"{label:28s} {ms:8.3f} ms/step", flush=True)


run("step only", False, False)
run("upload + step", True, False)
run("step + download", False, True)
run("upload + step + download", True, True)
