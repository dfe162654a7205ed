"""GPU: the pipelined transfer calls (nbody_set_bodies_async /
nbody_get_positions_async) give the same results as the synchronous calls,
with several input sets and steps in flight, and defer input validation to
nbody_sync."""
import numpy as np
import pytest

from workloads import generate

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def NB():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_sc_casselldahg24_b200 import NBody
    return NBody


def _inputs(n, k):
    return [generate(w, n, 20 + j) for j, w in zip(range(k), ["plummer", "disks", "clustered", "uniform"])]


@pytest.mark.parametrize("graph", [True, False])
def test_async_pipeline_equals_sync(NB, graph):
    import torch
    n, k = 20_011, 4
    sets = _inputs(n, k)
    ref = []
    sim = NB(n, 0.5, 1e-3, 1e-3, key_bits=16, use_graph=graph)
    for pos, vel, mass in sets:
        sim.set_bodies(pos, vel, mass)
        sim.step(2)
        ref.append(sim.get_positions())
    pinned = [tuple(torch.from_numpy(a).pin_memory() for a in s) for s in sets]
    outs = [torch.empty((n, 3), dtype=torch.float32).pin_memory() for _ in range(k)]
    sim2 = NB(n, 0.5, 1e-3, 1e-3, key_bits=16, use_graph=graph)
    keep = []
    for (hp, hv, hm), o in zip(pinned, outs):
        sim2.set_bodies_async(hp, hv, hm)
        keep.append((hp, hv, hm))
        sim2.step(2)
        sim2.get_positions_async(o)
    sim2.sync()
    for r, o in zip(ref, outs):
        assert (o.numpy() == r).all()


def test_async_device_buffers_and_deferred_validation(NB):
    import torch
    n = 4099
    pos, vel, mass = generate("plummer", n, 3)
    sim = NB(n, 0.5, 1e-3, 1e-3, key_bits=16)
    d = [torch.from_numpy(a).cuda() for a in (pos, vel, mass)]
    out = torch.empty((n, 3), dtype=torch.float32, device="cuda")
    sim.set_bodies_async(*d)
    sim.step(1)
    sim.get_positions_async(out)
    sim.sync()
    sim.set_bodies(pos, vel, mass)
    sim.step(1)
    assert (out.cpu().numpy() == sim.get_positions()).all()
    bad = mass.copy()
    bad[17] = 0.0
    sim.set_bodies_async(torch.from_numpy(pos).pin_memory(), torch.from_numpy(vel).pin_memory(),
                         torch.from_numpy(bad).pin_memory())
    with pytest.raises(Exception, match="async input set"):
        sim.sync()
    # the context stays usable after the deferred error
    sim.set_bodies(pos, vel, mass)
    sim.step(1)
    sim.sync()


@pytest.mark.parametrize("n", [1, 2, 33, 1025])
def test_async_small_and_ragged(NB, n):
    import torch
    pos, vel, mass = generate("uniform", n, 11)
    ref = NB(n, 0.5, 1e-3, 1e-3, key_bits=16)
    ref.set_bodies(pos, vel, mass)
    ref.compute_accel()
    a_ref = ref.get_accel()
    ref.set_bodies(pos, vel, mass)
    ref.step(3)
    x_ref = ref.get_positions()
    sim = NB(n, 0.5, 1e-3, 1e-3, key_bits=16)
    hp, hv, hm = (torch.from_numpy(a).pin_memory() for a in (pos, vel, mass))
    sim.set_bodies_async(hp, hv, hm)
    sim.compute_accel()
    assert (sim.get_accel() == a_ref).all()  # a synchronous getter after an async load
    sim.set_bodies_async(hp, hv, hm)
    sim.step(3)
    out = torch.empty((n, 3), dtype=torch.float32).pin_memory()
    sim.get_positions_async(out)
    sim.sync()
    assert (out.numpy() == x_ref).all()


def test_async_api_checks(NB):
    import torch
    n = 64
    pos, vel, mass = generate("uniform", n, 12)
    sim = NB(n, 0.5, 1e-3, 1e-3)
    out = torch.empty((n, 3), dtype=torch.float32).pin_memory()
    with pytest.raises(Exception):
        sim.get_positions_async(out)  # nothing loaded yet
    f64 = NB(n, 0.5, 1e-3, 1e-3, precision=64)
    with pytest.raises(ValueError):
        f64.set_bodies_async(pos, vel, mass)
    st = f64.lib.nbody_set_bodies_async(f64.h, None, None, None)
    assert st == -1  # NBODY_EINVAL
