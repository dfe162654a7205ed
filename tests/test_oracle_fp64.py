"""Pins for the oracle's FP64 mode (NEXT-2: the paper's own precision, P:272,
P:282), CPU only.

The fp64 mode evaluates the same step on fp64 bodies.  Each test checks it
against something other than itself: exact rationals, brute-force sums
(math.fsum) over each node's leaf range, exact min/max, the exact limit
theta = 0 == direct sum, closed forms, the BH partition of the bodies and the
leapfrog's second-order energy error.  P:NNN = line of
/root/reference/PAPER.md; [A#] = DESIGN.md reading.
"""
import math
from fractions import Fraction

import numpy as np
import pytest

from workloads import generate


def _rel_err(a, b):
    return np.linalg.norm(a - b, axis=1) / np.maximum(np.linalg.norm(b, axis=1), 1e-300)


def test_fp64_inputs_are_not_fp32_values():
    pos, vel, mass = generate("plummer", 1000, 3, np.float64)
    assert pos.dtype == np.float64 and (pos != pos.astype(np.float32).astype(np.float64)).mean() > 0.99


def test_fp64_bbox_is_exact_min_max(oracle):
    pos, _, _ = generate("disks", 5000, 4, np.float64)
    lo, hi = oracle.bbox(pos, 64)
    assert lo.dtype == np.float64 and (lo == pos.min(axis=0)).all() and (hi == pos.max(axis=0)).all()


@pytest.mark.parametrize("b", [1, 10, 16, 21])
def test_fp64_quantize_against_exact_rationals(oracle, b):
    """q = min(2^b - 1, floor((x - lo) 2^b / ext)) [A9][A16] on fp64 bodies:
    the oracle may differ from the exact rational floor only where the exact
    value lies within fp64 rounding of a cell boundary."""
    pos, _, _ = generate("plummer", 3000, 12, np.float64)
    q = oracle.quantize(pos, b, 64)
    lo, hi = pos.min(axis=0), pos.max(axis=0)
    ext = max(Fraction(float(hi[k])) - Fraction(float(lo[k])) for k in range(3))
    qmax = (1 << b) - 1
    for i in range(0, len(pos), 7):
        for k in range(3):
            v = (Fraction(float(pos[i, k])) - Fraction(float(lo[k]))) * (1 << b) / ext
            exact = min(qmax, math.floor(v))
            if q[i, k] != exact:
                assert abs(v - round(v)) <= Fraction(1, 10 ** 9) * max(1, v)
    widest = int(np.argmax(hi - lo))
    assert q[np.argmax(pos[:, widest]), widest] == qmax
    assert q[np.argmin(pos[:, widest]), widest] == 0


def test_fp64_mode_on_fp32_values_equals_fp32_mode(oracle):
    """fp32 bodies promoted to fp64 are the same numbers: keys, tree and
    forces of the two modes agree exactly (the fp64 mode adds no arithmetic
    of its own)."""
    pos, vel, mass = generate("clustered", 2000, 5)
    r32 = oracle.step(pos, vel, mass, theta=0.5, eps=1e-3, dt=1e-3, integrate=False)
    r64 = oracle.step(pos.astype(np.float64), vel.astype(np.float64), mass.astype(np.float64), theta=0.5,
                      eps=1e-3, dt=1e-3, integrate=False, precision=64)
    assert (r32.keys == r64.keys).all() and (r32.perm == r64.perm).all()
    assert (r32.acc == r64.acc).all() and (r32.count == r64.count).all()


@pytest.mark.parametrize("n", [1, 2, 5, 17, 1025])
def test_fp64_tree_matches_brute_force_ranges(oracle, n):
    """Node (l, j) aggregates leaves [j 2^l, min((j+1) 2^l, N)) (P:218,
    Fig. 4, [A6]): fp64 mass and COM vs math.fsum, exact AABB, and
    s^2 = (longest side)^2 of the fp64 box [A3]."""
    rng = np.random.default_rng(100 + n)
    pos = rng.normal(size=(n, 3))
    mass = rng.uniform(0.5, 2.0, n)
    t = oracle.Tree(pos, mass, 64)
    for l in range(t.L + 1):
        d = t.level(l)
        assert d.lo.dtype == np.float64
        for j in range(0, t.count(l), max(1, t.count(l) // 40)):
            a, b = j << l, min((j + 1) << l, n)
            M = math.fsum(mass[a:b])
            com = [math.fsum(Fraction(float(mass[i])) * Fraction(float(pos[i, k])) for i in range(a, b)) / M
                   for k in range(3)]
            assert d.M[j] == pytest.approx(M, rel=1e-14)
            assert np.allclose(d.com[j], np.array(com, float), rtol=0, atol=1e-13)
            assert (d.lo[j] == pos[a:b].min(axis=0)).all() and (d.hi[j] == pos[a:b].max(axis=0)).all()
            side = max(float(d.hi[j, k]) - float(d.lo[j, k]) for k in range(3))
            assert d.s2[j] == side * side


@pytest.mark.parametrize("name,n,seed", [("uniform", 1024, 1), ("plummer", 1025, 2), ("disks", 700, 3)])
def test_fp64_theta0_reproduces_direct_sum(oracle, name, n, seed):
    """theta = 0 opens every node: the BH sum is the direct sum (Eq. 1
    P:72) to 1e-12 relative on fp64 bodies."""
    pos, vel, mass = generate(name, n, seed, np.float64)
    r = oracle.step(pos, vel, mass, theta=0.0, eps=1e-3, dt=1e-3, integrate=False, precision=64)
    d = oracle.direct(r.tree.pos, r.tree.mass, 1e-3, precision=64)
    assert _rel_err(r.acc, d).max() <= 1e-12
    assert (r.count == n - 1).all()


def test_fp64_two_body_closed_form(oracle):
    pos = np.array([[0.1, 0.0, 0.0], [3.1, 4.0, 0.0]])
    mass = np.array([2.0, 0.5])
    eps = 0.25
    r = oracle.step(pos, np.zeros_like(pos), mass, theta=0.5, eps=eps, dt=1e-3, integrate=False, precision=64)
    acc = np.empty((2, 3))
    acc[r.ids] = r.acc
    dx = np.array([3.1 - 0.1, 4.0, 0.0])
    s = (float(dx @ dx) + eps * eps) ** 1.5
    assert np.allclose(acc[0], 0.5 * dx / s, rtol=1e-15, atol=0)
    assert np.allclose(acc[1], -2.0 * dx / s, rtol=1e-15, atol=0)


@pytest.mark.parametrize("theta", [0.5, 0.8])
def test_fp64_interaction_list_partitions_the_bodies(oracle, theta):
    """Each other body is covered by exactly one interaction;
    every accepted node passes the fp64 opening test and every proper
    ancestor fails it [A3][A20], evaluated here in exact rationals."""
    pos, vel, mass = generate("plummer", 500, 22, np.float64)
    r = oracle.step(pos, vel, mass, theta=theta, eps=1e-3, dt=1e-3, integrate=False, precision=64)
    t = r.tree
    levels = [t.level(l) for l in range(t.L + 1)]
    th2 = theta * theta

    def accept(lv, j, xk):
        d = [float(lv.com[j, k]) - float(xk[k]) for k in range(3)]
        d2 = float(Fraction(d[2]) ** 2 + Fraction(float(Fraction(d[1]) ** 2 + Fraction(d[0] * d[0]))))
        return float(lv.s2[j]) < th2 * d2

    for k in [0, 123, 499]:
        lst = t.force_list(theta, 1e-3, k)
        cover = np.zeros(t.n, np.int64)
        for l, j in lst:
            a, b = j << l, min((j + 1) << l, t.n)
            cover[a:b] += 1
            if l > 0:
                assert accept(levels[l], j, t.pos[k])
            for up in range(l + 1, t.L + 1):
                assert not accept(levels[up], j >> (up - l), t.pos[k])
        others = np.ones(t.n, bool)
        others[k] = False
        assert (cover[others] == 1).all()
        assert len(lst) == r.count[k]


def _kepler_energy_error64(oracle, dt, t_end, v=0.35):
    pos = np.array([[-0.5, 0, 0], [0.5, 0, 0]])
    mass = np.array([0.5, 0.5])
    a0 = np.array([[0.5, 0, 0], [-0.5, 0, 0]])
    vel = np.array([[0, -v, 0], [0, v, 0]]) - a0 * dt / 2
    ids = np.arange(2)
    x, u, m = pos, vel, mass
    e0, worst = None, 0.0
    for _ in range(int(round(t_end / dt))):
        r = oracle.step(x, u, m, ids, theta=0.5, eps=0.0, dt=dt, key_bits=16, precision=64)
        assert r.pos.dtype == np.float64
        xt = x[r.perm]
        vt = r.vel - 0.5 * dt * r.acc
        e = 0.5 * (r.mass * (vt ** 2).sum(axis=1)).sum() - 0.25 / np.linalg.norm(xt[0] - xt[1])
        x, u, m, ids = r.pos, r.vel, r.mass, r.ids
        e0 = e if e0 is None else e0
        worst = max(worst, abs(e - e0) / abs(e0))
    return worst


def test_fp64_leapfrog_energy_error_second_order(oracle):
    """Stormer-Verlet [A14] on fp64 state: bounded, O(dt^2) energy error."""
    e1 = _kepler_energy_error64(oracle, 0.04, 8.0)
    e2 = _kepler_energy_error64(oracle, 0.02, 8.0)
    e3 = _kepler_energy_error64(oracle, 0.01, 8.0)
    assert e1 < 0.05
    assert 3.5 < e1 / e2 < 4.5 and 3.5 < e2 / e3 < 4.5


def test_fp64_direct_sum_momentum(oracle):
    pos, _, mass = generate("plummer", 400, 27, np.float64)
    a = oracle.direct(pos, mass, 1e-3, precision=64)
    p = (mass[:, None] * a).sum(axis=0)
    assert np.abs(p).max() / (mass[:, None] * np.abs(a)).sum() < 1e-14
