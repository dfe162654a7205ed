"""Checkpoint / resume: nbody_set_state restores the slot-order
state written by nbody_get_state -- ids, slot order and the step counter --
so that stepping the restored context is bit-identical to stepping the
original (the stable sort's tie order, Alg. 7 P:201-212 [A10], and the
tree-reuse phase [A23] both depend on them), and the restored context's next
step matches the oracle run on the same state.
"""
import numpy as np
import pytest

from parity_utils import assert_acc_close
from paper_conf_sc_casselldahg24_b200._capi import NBodyError
from workloads import generate

pytestmark = pytest.mark.gpu

EPS, DT = 1e-3, 1e-3


@pytest.fixture(scope="module")
def NB():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_sc_casselldahg24_b200 import NBody
    return NBody


def _ids(vi):
    return vi[:, 3].view(np.int32).copy()


@pytest.mark.parametrize("sort_every,k_before,k_after", [(1, 2, 3), (3, 2, 4), (2, 3, 3)])
def test_resume_is_bit_identical(NB, sort_every, k_before, k_after):
    """A run interrupted after k_before steps and resumed in a NEW context
    (also with the other kind of CUDA-graph use) equals the uninterrupted
    run bit for bit: state, accelerations and interaction counts."""
    n = 20_011
    pos, vel, mass = generate("disks", n, 91)
    a = NB(n, 0.5, EPS, DT)
    a.set_option(7, sort_every)  # NBODY_OPT_SORT_EVERY
    a.set_bodies(pos, vel, mass)
    a.step(k_before)
    a.sync()
    pm, vi = a.get_state()
    steps = a.stats()["steps"]
    assert steps == k_before
    a.step(k_after)
    a.sync()
    pm_a, vi_a = a.get_state()

    b = NB(n, 0.5, EPS, DT, use_graph=False)
    b.set_option(7, sort_every)
    b.set_state(pm, vi, steps)
    assert b.stats()["steps"] == k_before
    b.step(k_after)
    b.sync()
    pm_b, vi_b = b.get_state()
    assert (pm_b.view(np.uint32) == pm_a.view(np.uint32)).all()
    assert (vi_b.view(np.uint32) == vi_a.view(np.uint32)).all()
    assert (b.get_accel().view(np.uint32) == a.get_accel().view(np.uint32)).all()
    assert (b.get_interactions() == a.get_interactions()).all()


def test_resume_from_device_arrays(NB):
    """The state may come from device memory (torch tensors)."""
    import torch
    n = 4099
    pos, vel, mass = generate("plummer", n, 92)
    a = NB(n, 0.5, EPS, DT)
    a.set_bodies(pos, vel, mass)
    a.step(1)
    pm, vi = a.get_state()
    a.step(1)
    b = NB(n, 0.5, EPS, DT)
    b.set_state(torch.from_numpy(pm).cuda(), torch.from_numpy(vi).cuda(), 1)
    b.step(1)
    assert (b.get_state()[0].view(np.uint32) == a.get_state()[0].view(np.uint32)).all()


def test_restored_step_matches_oracle(NB, oracle):
    """The restored context's next step on the checkpointed state is the
    oracle's step on that state (same slot order and ids): counts equal for
    every body, accelerations within the north-star tolerances."""
    n = 30_000
    pos, vel, mass = generate("clustered", n, 93)
    a = NB(n, 0.5, EPS, DT)
    a.set_bodies(pos, vel, mass)
    a.step(2)
    pm, vi = a.get_state()
    b = NB(n, 0.5, EPS, DT)
    b.set_state(pm, vi, 2)
    b.step(1)
    ref = oracle.step(pm[:, :3], vi[:, :3], pm[:, 3], _ids(vi), theta=0.5, eps=EPS, dt=DT)
    pm_b, vi_b = b.get_state()
    assert (_ids(vi_b) == ref.ids).all(), "slot order after the step differs from the oracle's stable sort"
    assert (b.get_interactions()[ref.ids] == ref.count).all()
    assert_acc_close(b.get_accel()[ref.ids], ref.acc)


def test_resume_keeps_the_tie_order(NB):
    """Heavy key ties (groups of 8 coincident bodies, equal Hilbert keys): the
    restored context's stable sort breaks them by the checkpointed slot
    order, exactly as the original run does."""
    n = 6000
    rng = np.random.default_rng(94)
    base = rng.uniform(-1, 1, (n // 8, 3)).astype(np.float32)
    pos = np.repeat(base, 8, axis=0)[rng.permutation(n)]  # groups of 8 coincident bodies: equal keys
    vel = np.zeros((n, 3), np.float32)
    mass = np.full(n, 1.0 / n, np.float32)
    a = NB(n, 0.5, EPS, 0.0)  # dt = 0: positions stay coincident
    a.set_bodies(pos, vel, mass)
    a.step(1)
    pm, vi = a.get_state()
    a.step(1)
    ids_a = _ids(a.get_state()[1])
    b = NB(n, 0.5, EPS, 0.0)
    b.set_state(pm, vi, 1)
    b.step(1)
    assert (_ids(b.get_state()[1]) == ids_a).all()


def test_set_state_rejects_invalid_states(NB):
    n = 1000
    pos, vel, mass = generate("uniform", n, 95)
    a = NB(n, 0.5, EPS, DT)
    a.set_bodies(pos, vel, mass)
    a.step(1)
    pm, vi = a.get_state()
    b = NB(n, 0.5, EPS, DT)
    dup = vi.copy()
    dup[5, 3] = dup[6, 3]                      # an id twice, another missing
    with pytest.raises(NBodyError, match="permutation"):
        b.set_state(pm, dup, 1)
    big = vi.copy()
    big[7, 3] = np.array([n], np.int32).view(np.float32)[0]
    with pytest.raises(NBodyError, match="permutation"):
        b.set_state(pm, big, 1)
    bad = pm.copy()
    bad[3, 3] = 0.0
    with pytest.raises(NBodyError, match="mass"):
        b.set_state(bad, vi, 1)
    nan = pm.copy()
    nan[2, 0] = np.nan
    with pytest.raises(NBodyError, match="non-finite"):
        b.set_state(nan, vi, 1)
    with pytest.raises(NBodyError):
        b.set_state(pm, vi, -1)
    with pytest.raises(NBodyError, match="no bodies"):
        b.step(1)
    b.set_state(pm, vi, 1)                     # a valid state loads again
    b.step(1)
    a.step(1)
    assert (b.get_state()[0].view(np.uint32) == a.get_state()[0].view(np.uint32)).all()


def test_resume_fp64_mode(NB):
    """NEXT-2 FP64 mode: nbody_set_state64 with the get_state64 layout."""
    n = 5003
    pos, vel, mass = generate("plummer", n, 96)
    a = NB(n, 0.5, EPS, DT, precision=64)
    a.set_bodies(pos.astype(np.float64), vel.astype(np.float64), mass.astype(np.float64))
    a.step(2)
    pm, vi = a.get_state64()
    a.step(2)
    b = NB(n, 0.5, EPS, DT, precision=64)
    b.set_state(pm, vi, 2)
    b.step(2)
    pa, va = a.get_state64()
    pb, vb = b.get_state64()
    assert (pa.view(np.uint64) == pb.view(np.uint64)).all() and (va.view(np.uint64) == vb.view(np.uint64)).all()
    frac = vi.copy()
    frac[0, 3] += 0.5                          # not an integer id
    with pytest.raises(NBodyError, match="permutation"):
        b.set_state(pm, frac, 2)


def test_resume_with_quadrupoles_and_tree_reuse(NB):
    """The restore carries everything a quadrupole, tree-reuse run needs: the
    resumed context steps bit-identically (moments are rebuilt from the
    restored state each step)."""
    n = 15_013
    pos, vel, mass = generate("clustered", n, 97)
    a = NB(n, 0.6, EPS, DT, multipole=2)
    a.set_option(7, 3)
    a.set_bodies(pos, vel, mass)
    a.step(4)
    pm, vi = a.get_state()
    steps = a.stats()["steps"]
    a.step(3)
    b = NB(n, 0.6, EPS, DT, multipole=2)
    b.set_option(7, 3)
    b.set_state(pm, vi, steps)
    b.step(3)
    assert (b.get_state()[0].view(np.uint32) == a.get_state()[0].view(np.uint32)).all()
    assert (b.get_accel().view(np.uint32) == a.get_accel().view(np.uint32)).all()
