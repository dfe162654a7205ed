"""Pins for the fp64 CPU oracle (oracle/), CPU only.

Each test checks the oracle against something other than itself: closed
forms, brute force on tiny inputs, library routines (numpy min/max/argsort,
math.fsum), curve invariants, or the exact limit (theta = 0 == direct sum).
P:NNN = line of /root/reference/PAPER.md; [A#] = DESIGN.md reading.
"""
import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

from workloads import generate

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


# ----------------------------------------------------------- O3: Hilbert ----
def test_hilbert_b1_golden_order(oracle):
    g = _golden("hilbert_b1_order.json")
    for key, cell in enumerate(g["cells_in_key_order"]):
        assert oracle.hilbert_index(*cell, 1) == key


def test_hilbert_b5_golden_examples(oracle):
    g = _golden("hilbert_b5_examples.json")
    for ex in g["examples"]:
        assert oracle.hilbert_index(*ex["cell"], g["b"]) == ex["key"]


def _all_cells(oracle, b):
    side = 1 << b
    inv = {}
    for x in range(side):
        for y in range(side):
            for z in range(side):
                inv[oracle.hilbert_index(x, y, z, b)] = (x, y, z)
    return inv


@pytest.mark.parametrize("b", [1, 2, 3, 4, 5])
def test_hilbert_bijection_and_unit_steps(oracle, b):
    """A Hilbert index is a bijection of the 8^b cells onto [0, 8^b) whose
    consecutive cells are face neighbours (Fig. 4)."""
    inv = _all_cells(oracle, b)
    assert sorted(inv) == list(range(8 ** b))
    cells = np.array([inv[k] for k in range(8 ** b)])
    steps = np.abs(np.diff(cells, axis=0)).sum(axis=1)
    assert (steps == 1).all()
    assert tuple(cells[0]) == (0, 0, 0)
    assert tuple(cells[-1]) == ((1 << b) - 1, 0, 0)


@pytest.mark.parametrize("b", [2, 3, 4])
def test_hilbert_octant_locality(oracle, b):
    """Every aligned run of 8^k consecutive indices fills one aligned cube of
    side 2^k -- the recursive-octant property that makes the curve Hilbert."""
    inv = _all_cells(oracle, b)
    cells = np.array([inv[k] for k in range(8 ** b)])
    for k in range(1, b):
        run = 8 ** k
        blocks = cells.reshape(-1, run, 3)
        lo, hi = blocks.min(axis=1), blocks.max(axis=1)
        assert ((hi - lo) == (1 << k) - 1).all()
        assert (lo % (1 << k) == 0).all()


def test_hilbert_b21_extremes(oracle):
    b = 21
    assert oracle.hilbert_index(0, 0, 0, b) == 0
    assert oracle.hilbert_index((1 << b) - 1, 0, 0, b) == 8 ** b - 1
    assert oracle.hilbert_index(1, 0, 0, 1) == 7


# --------------------------------------------------------- O1/O2: bbox, grid -
def test_bbox_matches_numpy(oracle):
    pos, _, _ = generate("disks", 5000, 11)
    lo, hi = oracle.bbox(pos)
    assert (lo == pos.min(axis=0)).all() and (hi == pos.max(axis=0)).all()


def test_paper_key_bits():
    from oracle import oracle as O
    # smallest b with 8^b >= N  [A8]
    for n, b in [(1, 1), (8, 1), (9, 2), (1024, 4), (10 ** 6, 7), (10 ** 7, 8), (10 ** 8, 9)]:
        assert O.paper_key_bits(n) == b


@pytest.mark.parametrize("b", [1, 4, 10, 16, 21])
def test_quantize_against_exact_rationals(oracle, b):
    """q_k = min(2^b - 1, floor((x_k - lo_k) 2^b / ext)); the fp64 oracle may
    differ from the exact rational floor only where the exact value lies
    within fp64 rounding of a cell boundary [A9][A16]."""
    pos, _, _ = generate("plummer", 3000, 12)
    q = oracle.quantize(pos, b)
    lo, hi = pos.min(axis=0), pos.max(axis=0)
    ext = max(Fraction(float(hi[k])) - Fraction(float(lo[k])) for k in range(3))
    qmax = (1 << b) - 1
    for i in range(0, len(pos), 7):
        for k in range(3):
            v = (Fraction(float(pos[i, k])) - Fraction(float(lo[k]))) * (1 << b) / ext
            exact = min(qmax, math.floor(v))
            if q[i, k] != exact:
                assert abs(v - round(v)) <= Fraction(1, 10 ** 9) * max(1, v)
    assert q.max() <= qmax
    # the body on the hi face of the widest axis lands in the last cell
    widest = int(np.argmax(hi.astype(np.float64) - lo.astype(np.float64)))
    assert q[np.argmax(pos[:, widest]), widest] == qmax
    assert q[np.argmin(pos[:, widest]), widest] == 0


def test_keys_compose_and_degenerate(oracle):
    pos, _, _ = generate("uniform", 2000, 13)
    b = 7
    q = oracle.quantize(pos, b)
    k = oracle.keys(pos, b)
    for i in range(0, 2000, 37):
        assert k[i] == oracle.hilbert_index(int(q[i, 0]), int(q[i, 1]), int(q[i, 2]), b)
    same = np.tile(np.float32([0.25, -1.5, 3.0]), (17, 1))
    assert (oracle.keys(same, 16) == 0).all()  # ext == 0 [A17]
    assert (oracle.keys(same[:1], 21) == 0).all()  # N == 1


# ------------------------------------------------------------------ O4 sort --
def test_sort_is_numpy_stable_argsort(oracle):
    rng = np.random.default_rng(5)
    for n, hi in [(1, 3), (7, 2), (1000, 5), (50000, 1 << 40), (4096, 1)]:
        k = rng.integers(0, hi, n).astype(np.uint64)
        assert (oracle.sort_perm(k) == np.argsort(k, kind="stable")).all()


# ------------------------------------------------------------------ O6 tree --
def _brute_node(pos, mass, l, j):
    a, b = j << l, min((j + 1) << l, len(mass))
    M = math.fsum(float(m) for m in mass[a:b])
    mx = [math.fsum(float(mass[i]) * float(pos[i, d]) for i in range(a, b)) for d in range(3)]
    return M, [v / M for v in mx], pos[a:b].min(axis=0), pos[a:b].max(axis=0)


@pytest.mark.parametrize("n", [1, 2, 3, 5, 17, 1023, 1025])
def test_tree_matches_brute_force_ranges(oracle, n):
    """Node (l, j) aggregates leaves [j 2^l, min((j+1) 2^l, N)) (Fig. 4
    P:226, [A6]): mass, centre of mass, AABB and (longest side)^2."""
    rng = np.random.default_rng(n)
    pos = rng.normal(size=(n, 3)).astype(np.float32)
    mass = rng.uniform(0.5, 2.0, n).astype(np.float32)
    t = oracle.Tree(pos, mass)
    assert t.L == (0 if n == 1 else math.ceil(math.log2(n)))
    for l in range(t.L + 1):
        assert t.count(l) == -(-n // (1 << l))
        d = t.level(l)
        for j in range(0, t.count(l), max(1, t.count(l) // 40)):
            M, com, lo, hi = _brute_node(pos, mass, l, j)
            assert d.M[j] == pytest.approx(M, rel=1e-14)
            assert np.allclose(d.com[j], com, rtol=0, atol=1e-13 * max(1.0, np.abs(pos).max()))
            assert (d.lo[j] == lo).all() and (d.hi[j] == hi).all()
            side = max(float(hi[k]) - float(lo[k]) for k in range(3))
            assert d.s2[j] == side * side
    root = t.level(t.L)
    assert root.M[0] == pytest.approx(math.fsum(mass.astype(float)), rel=1e-14)
    assert (root.lo[0] == pos.min(axis=0)).all() and (root.hi[0] == pos.max(axis=0)).all()


def test_tree_root_com_is_centroid_for_equal_masses(oracle):
    pos, _, mass = generate("uniform", 4097, 3)
    t = oracle.Tree(pos, mass)
    root = t.level(t.L)
    centroid = [math.fsum(pos[:, d].astype(float)) / len(pos) for d in range(3)]
    assert np.allclose(root.com[0], centroid, rtol=0, atol=1e-14)
    assert root.M[0] == pytest.approx(len(pos) * float(mass[0]), rel=1e-14)


def test_tree_children_boxes_nest(oracle):
    pos, _, mass = generate("clustered", 3000, 9)
    t = oracle.Tree(pos, mass)
    for l in range(1, t.L + 1):
        p, c = t.level(l), t.level(l - 1)
        idx = np.arange(c.lo.shape[0])
        par = idx // 2
        assert (p.lo[par] <= c.lo).all() and (p.hi[par] >= c.hi).all()


# ----------------------------------------------------------------- O7 force --
def _rel_err(a, b):
    return np.linalg.norm(a - b, axis=1) / np.maximum(np.linalg.norm(b, axis=1), 1e-300)


@pytest.mark.parametrize("name,n,seed", [("uniform", 1024, 1), ("plummer", 1025, 2), ("disks", 700, 3)])
def test_theta0_reproduces_direct_sum(oracle, name, n, seed):
    """theta = 0 opens every node: the BH sum is the direct sum (Eq. 1
    P:72) to 1e-12 relative (BASELINE.json north star)."""
    pos, vel, mass = generate(name, n, seed)
    r = oracle.step(pos, vel, mass, theta=0.0, eps=1e-3, dt=1e-3, integrate=False)
    d = oracle.direct(r.tree.pos, r.tree.mass, 1e-3)
    assert _rel_err(r.acc, d).max() <= 1e-12
    assert (r.count == n - 1).all()


def test_one_body_has_no_force(oracle):
    r = oracle.step(np.float32([[1, 2, 3]]), np.zeros((1, 3), np.float32), np.float32([1.0]),
                    theta=0.5, eps=0.0, dt=1e-3, integrate=False)
    assert (r.acc == 0).all() and (r.count == 0).all()


def test_two_body_closed_form(oracle):
    pos = np.float32([[0.0, 0.0, 0.0], [3.0, 4.0, 0.0]])
    mass = np.float32([2.0, 0.5])
    eps = 0.25
    r = oracle.step(pos, np.zeros_like(pos), mass, theta=0.5, eps=eps, dt=1e-3, integrate=False)
    ids = r.ids
    acc = np.empty((2, 3))
    acc[ids] = r.acc
    s = (25.0 + eps * eps) ** 1.5
    assert np.allclose(acc[0], 0.5 * np.array([3.0, 4.0, 0.0]) / s, rtol=1e-15, atol=0)
    assert np.allclose(acc[1], -2.0 * np.array([3.0, 4.0, 0.0]) / s, rtol=1e-15, atol=0)


def test_three_collinear_closed_form(oracle):
    pos = np.float32([[0, 0, 0], [1, 0, 0], [3, 0, 0]])
    mass = np.float32([1.0, 2.0, 4.0])
    t = oracle.Tree(pos, mass)  # positions already on a line; use as sorted slots
    acc, cnt = t.force(0.0, 0.0)
    assert np.allclose(acc[:, 0], [2 / 1 + 4 / 9, -1 / 1 + 4 / 4, -1 / 9 - 2 / 4], rtol=1e-15)
    assert (acc[:, 1:] == 0).all() and (cnt == 2).all()


def _fma(a, b, c):
    return float(Fraction(a) * Fraction(b) + Fraction(c))


def _accept(level, j, xk, th2):
    dx = float(level.com[j, 0]) - float(xk[0])
    dy = float(level.com[j, 1]) - float(xk[1])
    dz = float(level.com[j, 2]) - float(xk[2])
    d2 = _fma(dz, dz, _fma(dy, dy, dx * dx))
    return float(level.s2[j]) < th2 * d2


@pytest.mark.parametrize("theta", [0.3, 0.5, 0.8])
def test_interaction_list_partitions_the_bodies(oracle, theta):
    """Each body other than the target is covered by exactly one interaction
    (a leaf or one accepted node): the BH partition implied by P:106/P:112.
    Every accepted node passes the opening test; every proper ancestor of an
    entry fails it [A3][A20]."""
    pos, vel, mass = generate("plummer", 600, 21)
    r = oracle.step(pos, vel, mass, theta=theta, eps=1e-3, dt=1e-3, integrate=False)
    t = r.tree
    levels = [t.level(l) for l in range(t.L + 1)]
    th2 = theta * theta
    for k in [0, 1, 137, 299, 599]:
        lst = t.force_list(theta, 1e-3, k)
        cover = np.zeros(t.n, np.int64)
        xk = t.pos[k].astype(np.float64)
        for l, j in lst:
            a, b = j << l, min((j + 1) << l, t.n)
            cover[a:b] += 1
            if l > 0:
                assert _accept(levels[l], j, xk, th2)
            for up in range(l + 1, t.L + 1):
                assert not _accept(levels[up], j >> (up - l), xk, th2)
        others = np.ones(t.n, bool)
        others[k] = False
        assert (cover[others] == 1).all()
        assert cover[k] in (0, 1)
        if theta < 1 / math.sqrt(3):
            assert cover[k] == 0  # [A4] cannot accept a node containing the target
        assert len(lst) == r.count[k]


def _skip_walk(levels, n, L, xk, th2, k):
    """[A7] stackless walk over the balanced BVH read as a skip list (P:222,
    P:245): cursor (l, s), s = first leaf covered; open -> l-1; done ->
    s += 2^l, l = min(ctz(s), L)."""
    out = []
    l, s = L, 0
    while True:
        done = True
        if l == 0:
            if s != k:
                out.append((0, s))
        elif _accept(levels[l], s >> l, xk, th2):
            out.append((l, s >> l))
        else:
            l -= 1
            done = False
        if done:
            s += 1 << l
            if s >= n:
                return out
            l = min((s & -s).bit_length() - 1, L)


@pytest.mark.parametrize("n", [2, 5, 300, 513])
def test_recursive_dfs_equals_skip_list_walk(oracle, n):
    pos, vel, mass = generate("clustered", n, 22)
    r = oracle.step(pos, vel, mass, theta=0.5, eps=1e-3, dt=1e-3, integrate=False)
    t = r.tree
    levels = [t.level(l) for l in range(t.L + 1)]
    for k in sorted({0, n // 2, n - 1}):
        lst = [tuple(e) for e in t.force_list(0.5, 1e-3, k)]
        assert lst == _skip_walk(levels, n, t.L, t.pos[k].astype(np.float64), 0.25, k)


def test_bh_error_shrinks_with_theta(oracle):
    pos, vel, mass = generate("uniform", 4096, 23)
    exact = None
    rms = []
    for theta in (0.8, 0.5, 0.3):
        r = oracle.step(pos, vel, mass, theta=theta, eps=1e-3, dt=1e-3, integrate=False)
        if exact is None:
            exact = oracle.direct(r.tree.pos, r.tree.mass, 1e-3)
        rms.append(float(np.sqrt(np.mean(_rel_err(r.acc, exact) ** 2))))
    assert rms[0] > rms[1] > rms[2]
    assert rms[1] < 2e-2


def test_far_cluster_monopole_error_is_second_order(oracle):
    """A cluster of 2^8 bodies plus one target placed in the last Hilbert cell
    (x = max, y = z = min -> key 8^b - 1, the curve's end point): the root's
    left child is exactly the cluster, so with theta = 1 the target's list is
    that single monopole and its error vs the direct sum is the
    quadrupole term, O((s/d)^2)."""
    rng = np.random.default_rng(4)
    blob = rng.uniform(-0.5, 0.5, (256, 3)) * [1.0, 2.0, 0.5]
    errs = []
    for d in (8.0, 16.0, 32.0, 64.0):
        pos = np.vstack([blob, [[d, -1.0, -0.25]]]).astype(np.float32)
        mass = np.full(len(pos), 1.0 / 256, np.float32)
        r = oracle.step(pos, np.zeros_like(pos), mass, theta=1.0, eps=0.0, dt=1e-3, integrate=False)
        slot = int(np.nonzero(r.ids == 256)[0][0])
        assert slot == 256 and r.count[slot] == 1
        exact = oracle.direct(pos, mass, 0.0, targets=[256])[0]
        errs.append(np.linalg.norm(r.acc[slot] - exact) / np.linalg.norm(exact))
    assert errs[0] < 1e-2
    for a, b in zip(errs, errs[1:]):
        assert 3.6 < a / b < 4.4


def test_plummer_mean_radial_acceleration(oracle):
    """Mean radial acceleration of a Plummer sphere (G = M = 1, a = 3 pi/16)
    follows -r / (r^2 + a^2)^(3/2) within sampling noise."""
    n = 1 << 15
    pos, vel, mass = generate("plummer", n, 24)
    r = oracle.step(pos, vel, mass, theta=0.5, eps=1e-4, dt=1e-3, integrate=False)
    x = r.tree.pos.astype(np.float64)
    rad = np.linalg.norm(x, axis=1)
    ar = (r.acc * x).sum(axis=1) / rad
    a = 3 * math.pi / 16
    for lo, hi in [(0.2, 0.4), (0.4, 0.7), (0.7, 1.0), (1.0, 1.5)]:
        m = (rad >= lo) & (rad < hi)
        model = -(rad[m] / (rad[m] ** 2 + a * a) ** 1.5).mean()
        assert abs(ar[m].mean() / model - 1) < 0.06


# ---------------------------------------------------------------- D direct --
def test_direct_sum_momentum_conservation(oracle):
    pos, _, mass = generate("clustered", 2000, 25)
    acc = oracle.direct(pos, mass, 1e-3)
    f = mass[:, None].astype(float) * acc
    assert np.linalg.norm(f.sum(axis=0)) / np.linalg.norm(f, axis=1).sum() < 1e-14


def test_direct_sum_coincident_bodies_without_softening(oracle):
    pos = np.float32([[0, 0, 0], [0, 0, 0], [2, 0, 0]])
    mass = np.float32([1, 1, 1])
    acc = oracle.direct(pos, mass, 0.0)
    assert np.allclose(acc[0], [0.25, 0, 0]) and np.allclose(acc[2], [-0.5, 0, 0])


# --------------------------------------------------------------- O8 leapfrog -
def _kepler_energy_error(oracle, dt, t_end, v=0.35):
    """Two bodies (m = 1/2 each, separation 1) on an eccentric bound orbit;
    returns max |E(t) - E(0)| / |E(0)| with E evaluated at force times:
    x_t (pre-drift) and v_t = v_{t+1/2} - a(x_t) dt / 2."""
    pos = np.float32([[-0.5, 0, 0], [0.5, 0, 0]])
    mass = np.float32([0.5, 0.5])
    a0 = np.array([[0.5, 0, 0], [-0.5, 0, 0]])
    vel = (np.array([[0, -v, 0], [0, v, 0]]) - a0 * dt / 2).astype(np.float32)  # v_{-1/2}
    ids = np.arange(2)
    x, u, m = pos, vel, mass
    e0, worst = None, 0.0
    for _ in range(int(round(t_end / dt))):
        r = oracle.step(x, u, m, ids, theta=0.5, eps=0.0, dt=dt, key_bits=16)
        xt = x[r.perm].astype(float)
        vt = r.vel.astype(float) - 0.5 * dt * r.acc
        e = 0.5 * (r.mass.astype(float) * (vt ** 2).sum(axis=1)).sum() - 0.25 / np.linalg.norm(xt[0] - xt[1])
        x, u, m, ids = r.pos, r.vel, r.mass, r.ids
        e0 = e if e0 is None else e0
        worst = max(worst, abs(e - e0) / abs(e0))
    return worst


def test_leapfrog_energy_error_second_order(oracle):
    """Stormer-Verlet (ref [12]) [A14]: bounded energy error, O(dt^2)."""
    e1 = _kepler_energy_error(oracle, 0.04, 8.0)
    e2 = _kepler_energy_error(oracle, 0.02, 8.0)
    e3 = _kepler_energy_error(oracle, 0.01, 8.0)
    assert e1 < 0.05
    assert 3.5 < e1 / e2 < 4.5 and 3.5 < e2 / e3 < 4.5


def test_leapfrog_conserves_momentum_with_exact_forces(oracle):
    pos, vel, mass = generate("plummer", 300, 26)
    p0 = (mass[:, None].astype(float) * vel.astype(float)).sum(axis=0)
    ids = np.arange(300)
    x, u, m = pos, vel, mass
    for _ in range(5):
        r = oracle.step(x, u, m, ids, theta=0.0, eps=1e-2, dt=1e-3)
        x, u, m, ids = r.pos, r.vel, r.mass, r.ids
    p1 = (m[:, None].astype(float) * u.astype(float)).sum(axis=0)
    scale = (mass[:, None] * np.abs(vel)).sum()
    assert np.abs(p1 - p0).max() / scale < 1e-6


# ------------------------------------------------- NEXT-3(iii) tree reuse ---
def test_tree_reuse_on_sorted_state_equals_resort(oracle):
    """resort=False on bodies already in Hilbert order (the previous step's
    output, positions unchanged) is the same step as a fresh sort."""
    pos, vel, mass = generate("plummer", 3000, 81)
    r0 = oracle.step(pos, vel, mass, theta=0.5, eps=1e-3, dt=0.0)
    a = oracle.step(r0.pos, r0.vel, r0.mass, r0.ids, theta=0.5, eps=1e-3, dt=1e-3)
    b = oracle.step(r0.pos, r0.vel, r0.mass, r0.ids, theta=0.5, eps=1e-3, dt=1e-3, resort=False)
    assert (a.perm == np.arange(3000)).all()
    assert (a.acc == b.acc).all() and (a.count == b.count).all() and (a.pos == b.pos).all()


def test_tree_reuse_keeps_exactness_properties(oracle):
    """Any leaf order gives a valid BVH: theta = 0 is still the direct sum and
    every list still partitions the other bodies."""
    pos, vel, mass = generate("uniform", 700, 82)  # unsorted array order
    r = oracle.step(pos, vel, mass, theta=0.0, eps=1e-3, dt=1e-3, integrate=False, resort=False)
    assert (r.ids == np.arange(700)).all()
    d = oracle.direct(pos, mass, 1e-3)
    assert _rel_err(r.acc, d).max() <= 1e-12 and (r.count == 699).all()
    r = oracle.step(pos, vel, mass, theta=0.5, eps=1e-3, dt=1e-3, integrate=False, resort=False)
    for k in (0, 350, 699):
        cover = np.zeros(700, np.int64)
        for l, j in r.tree.force_list(0.5, 1e-3, k):
            cover[j << l: min((j + 1) << l, 700)] += 1
        assert cover[k] == 0 and (np.delete(cover, k) == 1).all()


# --------------------------------------------------- NEXT-4 quadrupoles ------
def test_second_moments_match_brute_force(oracle):
    """[A24] S = sum m (x - com)(x - com)^T over each node's leaf range."""
    rng = np.random.default_rng(91)
    n = 777
    pos = rng.normal(size=(n, 3)).astype(np.float32)
    mass = rng.uniform(0.5, 2.0, n).astype(np.float32)
    t = oracle.Tree(pos, mass)
    ii, jj = [0, 1, 2, 0, 0, 1], [0, 1, 2, 1, 2, 2]
    for l in range(0, t.L + 1):
        S = t.level_quad(l)
        com = t.level(l).com
        for j in range(0, t.count(l), max(1, t.count(l) // 25)):
            a, b = j << l, min((j + 1) << l, n)
            y = pos[a:b].astype(float) - com[j]
            m = mass[a:b].astype(float)
            scale = math.fsum(m * (y ** 2).sum(axis=1)) + 1e-300
            for q in range(6):
                ref = math.fsum(m * y[:, ii[q]] * y[:, jj[q]])
                assert abs(S[j, q] - ref) <= 1e-12 * scale


def test_quadrupole_two_point_closed_form(oracle):
    """Masses m/2 at c -+ (s, 0, 0), target on the axis at distance D: the
    monopole is off by 3 s^2/D^2, the quadrupole term removes it (what is left
    is O(s^4/D^4))."""
    s = 0.25
    for D in (4.0, 8.0):
        pos = np.float32([[-s, 0, 0], [s, 0, 0], [D, 0, 0]])  # target last in Hilbert order (cell 2^b-1,0,0)
        mass = np.float32([0.5, 0.5, 1e-6])
        exact = 0.5 / (D - s) ** 2 + 0.5 / (D + s) ** 2
        mono = oracle.step(pos, np.zeros_like(pos), mass, theta=1.0, eps=0.0, dt=0.0, integrate=False)
        quad = oracle.step(pos, np.zeros_like(pos), mass, theta=1.0, eps=0.0, dt=0.0, integrate=False, quad=True)
        k = int(np.nonzero(mono.ids == 2)[0][0])
        assert mono.count[k] == 1  # one accepted node: the pair
        em = abs(-mono.acc[k, 0] - exact) / exact
        eq = abs(-quad.acc[k, 0] - exact) / exact
        assert em == pytest.approx(3 * s * s / D ** 2, rel=0.2)
        assert eq < 10 * (s / D) ** 4


def test_quadrupole_far_cluster_is_third_order(oracle):
    rng = np.random.default_rng(4)
    blob = rng.uniform(-0.5, 0.5, (256, 3)) * [1.0, 2.0, 0.5]
    em, eq = [], []
    for d in (8.0, 16.0, 32.0):
        pos = np.vstack([blob, [[d, -1.0, -0.25]]]).astype(np.float32)
        mass = np.full(len(pos), 1.0 / 256, np.float32)
        exact = oracle.direct(pos, mass, 0.0, targets=[256])[0]
        for q, out in ((False, em), (True, eq)):
            r = oracle.step(pos, np.zeros_like(pos), mass, theta=1.0, eps=0.0, dt=0.0, integrate=False, quad=q)
            assert r.count[256] == 1
            out.append(np.linalg.norm(r.acc[256] - exact) / np.linalg.norm(exact))
    assert all(q < m / 10 for q, m in zip(eq, em))
    for a, b in zip(eq, eq[1:]):
        assert 6.0 < a / b < 18.0  # at least third order


def test_quadrupole_improves_accuracy_same_lists(oracle):
    pos, vel, mass = generate("uniform", 4096, 92)
    m = oracle.step(pos, vel, mass, theta=0.6, eps=1e-3, dt=0.0, integrate=False)
    q = oracle.step(pos, vel, mass, theta=0.6, eps=1e-3, dt=0.0, integrate=False, quad=True)
    assert (m.count == q.count).all()  # the opening test does not change
    exact = oracle.direct(m.tree.pos, m.tree.mass, 1e-3)
    rm = np.sqrt(np.mean(_rel_err(m.acc, exact) ** 2))
    rq = np.sqrt(np.mean(_rel_err(q.acc, exact) ** 2))
    assert rq < 0.5 * rm
    z = oracle.step(pos, vel, mass, theta=0.0, eps=1e-3, dt=0.0, integrate=False, quad=True)
    assert _rel_err(z.acc, exact).max() <= 1e-12
