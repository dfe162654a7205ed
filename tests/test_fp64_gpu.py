"""GPU parity of the FP64 mode (NEXT-2; the paper's own precision, P:272,
P:282) against the oracle's fp64 mode on the same seeded fp64 inputs.

Bars: Hilbert keys, permutation and sorted state bit-exact; node records
(fp64 COM, s^2, mass, fp64 boxes) bit-exact on every level; interaction
counts equal; accelerations agree to fp64 rounding: the only differences are
the summation order and rsqrt vs 1/(r2 sqrt(r2)) (a few ulp per term), so
the bar is RMS relative 1e-12 and 1e-9 for every body.
"""
import numpy as np
import pytest

from workloads import generate

pytestmark = pytest.mark.gpu

EPS = 1e-3
DT = 1e-3


@pytest.fixture(scope="module")
def NB():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_sc_casselldahg24_b200 import NBody
    return NBody


def _rel(a, b):
    return np.linalg.norm(a - b, axis=1) / np.maximum(np.linalg.norm(b, axis=1), 1e-300)


def _check(NB, oracle, name, n, seed, theta=0.5, eps=EPS, levels=True):
    pos, vel, mass = generate(name, n, seed, np.float64)
    sim = NB(n, theta, eps, DT, precision=64)
    sim.set_bodies(pos, vel, mass)
    sim.compute_accel()
    ref = oracle.step(pos, vel, mass, theta=theta, eps=eps, dt=DT, integrate=False, precision=64)
    assert (sim.debug_keys() == ref.keys).all()
    assert (sim.debug_perm() == ref.perm).all()
    pm, vi = sim.get_state64()
    assert (pm[:, :3] == ref.pos).all() and (pm[:, 3] == ref.mass).all()
    assert (vi[:, 3].astype(np.int64) == ref.ids).all()
    if levels:
        for l in range(1, ref.tree.L + 1):
            pred, rec, _ = sim.debug_level(l)
            rec64, box64 = sim.debug_level64(l)
            d = ref.tree.level(l)
            assert (pred[:, :3] == d.com).all() and (pred[:, 3] == d.s2).all(), f"pred level {l}"
            assert (rec64[:, :3] == d.com).all() and (rec64[:, 3] == d.M).all(), f"rec64 level {l}"
            assert (box64[:, :3] == d.lo).all() and (box64[:, 3:] == d.hi).all(), f"box level {l}"
    acc = sim.get_accel64()[ref.ids]
    cnt = sim.get_interactions()[ref.ids]
    assert (cnt == ref.count).all()
    err = _rel(acc, ref.acc)
    assert np.sqrt(np.mean(err ** 2)) <= 1e-12 and err.max() <= 1e-9, (np.sqrt(np.mean(err ** 2)), err.max())
    return sim, ref


@pytest.mark.parametrize("name,n,seed", [("uniform", 1024, 1), ("plummer", 4099, 2), ("disks", 20_000, 3),
                                         ("clustered", 33_333, 4)])
def test_fp64_force_pass_matches_oracle(NB, oracle, name, n, seed):
    _check(NB, oracle, name, n, seed)


@pytest.mark.parametrize("theta", [0.3, 0.8])
def test_fp64_theta_sweep(NB, oracle, theta):
    _check(NB, oracle, "plummer", 10_007, 5, theta=theta, levels=False)


def test_fp64_unsoftened(NB, oracle):
    _check(NB, oracle, "uniform", 3000, 6, eps=0.0, levels=False)


def test_fp64_theta0_is_direct_sum(NB, oracle):
    """theta = 0: the GPU's fp64 BH sum is the fp64 direct sum (Eq. 1)."""
    n = 2000
    pos, vel, mass = generate("plummer", n, 7, np.float64)
    sim = NB(n, 0.0, EPS, DT, precision=64)
    sim.set_bodies(pos, vel, mass)
    sim.compute_accel()
    d = oracle.direct(pos, mass, EPS, precision=64)
    assert _rel(sim.get_accel64(), d).max() <= 1e-12
    assert (sim.get_interactions() == n - 1).all()


def test_fp64_steps_track_oracle(NB, oracle):
    """Three fp64 steps (re-sort every step) stay within fp64 rounding of the
    oracle's trajectory and leave keys/orders identical."""
    n = 8000
    pos, vel, mass = generate("disks", n, 8, np.float64)
    sim = NB(n, 0.5, EPS, DT, precision=64)
    sim.set_bodies(pos, vel, mass)
    x, v, m, ids = pos, vel, mass, np.arange(n)
    for _ in range(3):
        r = oracle.step(x, v, m, ids, theta=0.5, eps=EPS, dt=DT, precision=64)
        x, v, m, ids = r.pos, r.vel, r.mass, r.ids
    sim.step(3)
    xg = sim.get_positions64()
    xo = np.empty_like(xg)
    xo[ids] = x
    vg = sim.get_velocities64()
    vo = np.empty_like(vg)
    vo[ids] = v
    assert np.abs(xg - xo).max() <= 1e-12 * max(1.0, np.abs(xo).max())
    assert np.abs(vg - vo).max() <= 1e-12 * max(1.0, np.abs(vo).max())
    # the fp32 getters round the fp64 state
    assert (sim.get_positions() == xg.astype(np.float32)).all()


def test_fp64_mode_api_checks(NB):
    from paper_conf_sc_casselldahg24_b200 import _capi
    n = 100
    pos, vel, mass = generate("uniform", n, 9, np.float64)
    s = NB(n, 0.5, EPS, DT, precision=64)
    p32, v32, m32 = pos.astype(np.float32), vel.astype(np.float32), mass.astype(np.float32)
    assert s.lib.nbody_set_bodies(s.h, p32.ctypes.data, v32.ctypes.data, m32.ctypes.data) == _capi.NBODY_EINVAL
    with pytest.raises(_capi.NBodyError):
        s.set_option(_capi.NBODY_OPT_MULTIPOLE, 2)
    with pytest.raises(_capi.NBodyError):
        s.set_option(_capi.NBODY_OPT_TRAVERSAL, 1)
    bad = mass.copy()
    bad[3] = -1.0
    with pytest.raises(_capi.NBodyError):
        s.set_bodies(pos, vel, bad)
    t = NB(n, 0.5, EPS, DT)  # precision 32
    assert t.lib.nbody_set_bodies64(t.h, pos.ctypes.data, vel.ctypes.data, mass.ctypes.data) == _capi.NBODY_EINVAL
    with pytest.raises(_capi.NBodyError):
        t.get_accel64()
    # switching back to 32 restores the fp32 path
    s.set_option(_capi.NBODY_OPT_PRECISION, 32)
    s.precision = 32
    s.set_bodies(pos.astype(np.float32), vel.astype(np.float32), mass.astype(np.float32))
    s.compute_accel()
    assert np.isfinite(s.get_accel()).all()


def test_fp64_large_sampled(NB, oracle):
    """N = 10^6 Plummer (config 2 size) in fp64: keys/perm bit-exact, counts
    and accelerations of 3000 sampled targets against the oracle."""
    n = 1_000_000
    pos, vel, mass = generate("plummer", n, 2, np.float64)
    sim = NB(n, 0.5, EPS, DT, precision=64)
    sim.set_bodies(pos, vel, mass)
    sim.compute_accel()
    rng = np.random.default_rng(11)
    tg = np.sort(rng.choice(n, 3000, replace=False)).astype(np.int64)
    ref = oracle.step(pos, vel, mass, theta=0.5, eps=EPS, dt=DT, integrate=False, targets=tg, precision=64)
    assert (sim.debug_keys() == ref.keys).all() and (sim.debug_perm() == ref.perm).all()
    ids = ref.ids[tg]
    acc = sim.get_accel64()[ids]
    cnt = sim.get_interactions()[ids]
    assert (cnt == ref.count).all()
    err = _rel(acc, ref.acc)
    assert np.sqrt(np.mean(err ** 2)) <= 1e-12 and err.max() <= 1e-9
