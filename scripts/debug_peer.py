import sys, os, time
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np
from paper_conf_sc_casselldahg24_b200 import NBody
from workloads import generate
world, n, name, trav, graph = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3], int(sys.argv[4]), int(sys.argv[5])
pos, vel, mass = generate(name, n, 82)
ranks = [NBody(n, 0.5, 1e-3, 1e-3, traversal=trav, use_graph=bool(graph), device=0) for _ in range(world)]
NBody.attach_peers_local(ranks)
for s in ranks:
    s.set_bodies(pos, vel, mass)
t0 = time.time()
for k in range(3):
    for s in ranks:
        s.step(1)
    for s in ranks:
        s.sync()
print("ok", sys.argv[1:], time.time() - t0)
