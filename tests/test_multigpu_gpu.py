"""Multi-GPU path on one GPU.

NCCL cannot host two ranks on one device, so the G-rank step is emulated with
G contexts on the same GPU (nbody_set_partition) whose owned slices are
exchanged with nbody_copy_owned after each step -- exactly the data the NCCL
all-gather moves.  The bar is bit-identity with the single-context run.  A
world-1 NCCL communicator exercises the NCCL calls inside the captured graph.
"""
import numpy as np
import pytest

from workloads import generate

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def NB():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_sc_casselldahg24_b200 import NBody
    return NBody


def _single(NB, pos, vel, mass, steps):
    s = NB(len(pos), 0.5, 1e-3, 1e-3)
    s.set_bodies(pos, vel, mass)
    s.step(steps)
    return s


@pytest.mark.parametrize("world,n", [(2, 20_000), (3, 10_007), (8, 40_000), (8, 100)])
def test_emulated_partition_is_bit_identical(NB, world, n):
    steps = 3
    pos, vel, mass = generate("disks", n, 40 + world)
    ref = _single(NB, pos, vel, mass, steps)
    ranks = [NB(n, 0.5, 1e-3, 1e-3) for _ in range(world)]
    for r, s in enumerate(ranks):
        s.set_partition(r, world)
        s.set_bodies(pos, vel, mass)
    owned = [s.partition()[2:] for s in ranks]
    assert owned[0][0] == 0 and owned[-1][1] == n
    for _ in range(steps):
        for s in ranks:
            s.step(1)
        # after the force pass: owned accelerations assemble the full field
        for dst in ranks:
            for src in ranks:
                if src is not dst:
                    dst.copy_owned_from(src)
    x_ref, v_ref, a_ref = ref.get_positions(), ref.get_velocities(), ref.get_accel()
    c_ref = ref.get_interactions()
    total = 0
    a = np.full_like(a_ref, np.nan)
    c = np.zeros_like(c_ref)
    for s in ranks:
        assert (s.get_positions() == x_ref).all()
        assert (s.get_velocities() == v_ref).all()
        s.get_accel(a)  # writes only the owned bodies
        s.get_interactions(c)
        total += s.stats()["interactions"]
    assert (a == a_ref).all() and (c == c_ref).all()
    assert total == ref.stats()["interactions"]


def test_nccl_world1_matches_plain(NB):
    from paper_conf_sc_casselldahg24_b200 import _capi, dist
    if not _capi.load().nbody_has_nccl():
        pytest.skip("library built without NCCL")
    n = 30_000
    pos, vel, mass = generate("plummer", n, 50)
    ref = _single(NB, pos, vel, mass, 4)
    s = NB(n, 0.5, 1e-3, 1e-3)
    s.attach_nccl(dist.new_unique_id(), 0, 1)
    s.set_bodies(pos, vel, mass)
    s.step(4)
    assert (s.get_positions() == ref.get_positions()).all()
    assert (s.get_accel() == ref.get_accel()).all()
    assert (s.get_interactions() == ref.get_interactions()).all()
