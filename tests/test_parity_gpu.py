"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle on
the same seeded inputs.

Bars: Hilbert keys and sort permutation bit-exact; BVH
node records (fp64 com and s^2, fp32 monopole, fp32 box) bit-exact, which
implies the north star's 1e-6 node tolerance; interaction counts per body
equal; accelerations within 1e-4 RMS relative and 1e-2 for every body.
"""
import numpy as np
import pytest

from parity_utils import assert_acc_close, rel_errors
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


def _run_gpu(NB, pos, vel, mass, theta, key_bits, eps=EPS, traversal=0):
    sim = NB(len(pos), theta, eps, DT, key_bits=key_bits, traversal=traversal)
    sim.set_bodies(pos, vel, mass)
    sim.compute_accel()
    return sim


def _check_pass(NB, oracle, pos, vel, mass, theta=0.5, key_bits=16, eps=EPS, targets=None, levels=True,
                traversal=0):
    """One force pass on both sides; returns (gpu sim, oracle result)."""
    n = len(pos)
    sim = _run_gpu(NB, pos, vel, mass, theta, key_bits, eps, traversal)
    ref = oracle.step(pos, vel, mass, theta=theta, eps=eps, dt=DT, key_bits=key_bits, integrate=False,
                      targets=targets)
    # K2 / K3: keys and permutation bit-exact
    assert (sim.debug_keys() == ref.keys).all()
    assert (sim.debug_perm() == ref.perm).all()
    # sorted state: slot order of the GPU equals the oracle's
    pm, vi = sim.get_state()
    assert (pm[:, :3] == ref.pos).all() and (pm[:, 3] == ref.mass).all()
    ids = vi[:, 3].view(np.int32)
    assert (ids == ref.ids).all()
    # K5: node records bit-exact, every level
    if levels:
        for l in range(1, ref.tree.L + 1):
            pred, rec, box = sim.debug_level(l)
            d = ref.tree.level(l)
            assert (pred[:, :3] == d.com).all(), f"com level {l}"
            assert (pred[:, 3] == d.s2).all(), f"s2 level {l}"
            assert (rec[:, :3] == d.c32).all() and (rec[:, 3] == d.m32).all(), f"rec level {l}"
            assert (box[:, :3] == d.lo).all() and (box[:, 3:] == d.hi).all(), f"box level {l}"
    # K6: interaction counts equal, accelerations within tolerance
    acc_id = sim.get_accel()
    cnt_id = sim.get_interactions()
    tg = ref.targets
    ids_t = ref.ids[tg]
    assert (cnt_id[ids_t] == ref.count).all(), "interaction counts differ"
    assert_acc_close(acc_id[ids_t], ref.acc)
    return sim, ref


CASES = [
    ("uniform", 1024, 1, 0.5, 16),     # config 1
    ("uniform", 1024, 1, 0.0, 16),     # theta = 0: direct sum
    ("plummer", 20_000, 2, 0.5, 16),
    ("disks", 30_001, 3, 0.5, 16),     # ragged: odd N
    ("clustered", 25_000, 4, 0.8, 16),
    ("clustered", 25_000, 4, 0.3, 10),  # u32 keys
    ("plummer", 12_345, 5, 0.5, 0),    # paper grid rule (b = 5): heavy key ties
    ("disks", 9_000, 6, 0.5, 21),      # 63-bit keys
    ("uniform", 4097, 7, 0.5, 1),      # 3-bit keys: 8 cells, ties everywhere
]


@pytest.mark.parametrize("bits", list(range(1, 22)))
def test_keys_every_grid_resolution(NB, oracle, bits):
    """K2's table-driven Skilling automaton equals the oracle's transform at
    every b (odd b takes the single-level table at the top), and K3's
    permutation follows."""
    pos, vel, mass = generate("clustered", 6001, 8)
    sim = _run_gpu(NB, pos, vel, mass, 0.5, bits)
    ref = oracle.step(pos, vel, mass, theta=0.5, eps=EPS, dt=DT, key_bits=bits, integrate=False,
                      targets=np.array([0, 6000]))
    assert (sim.debug_keys() == ref.keys).all()
    assert (sim.debug_perm() == ref.perm).all()


@pytest.mark.parametrize("name,n,seed,theta,bits", CASES)
def test_force_pass_parity(NB, oracle, name, n, seed, theta, bits):
    pos, vel, mass = generate(name, n, seed)
    _check_pass(NB, oracle, pos, vel, mass, theta=theta, key_bits=bits)


@pytest.mark.parametrize("n", [1, 2, 3, 5, 31, 32, 33, 63, 65, 257])
def test_small_and_ragged_n(NB, oracle, n):
    pos, vel, mass = generate("plummer", n, 100 + n)
    _check_pass(NB, oracle, pos, vel, mass, theta=0.5)


def test_all_bodies_coincident(NB, oracle):
    n = 1000
    pos = np.tile(np.float32([0.5, -0.25, 2.0]), (n, 1))
    vel = np.zeros_like(pos)
    mass = np.full(n, 1.0 / n, np.float32)
    sim, ref = _check_pass(NB, oracle, pos, vel, mass, theta=0.5, eps=1e-2)
    assert (sim.debug_keys() == 0).all()


def test_zero_softening_with_coincident_pairs(NB, oracle):
    pos, vel, mass = generate("uniform", 2000, 8)
    pos[1000:1010] = pos[0]  # coincident with body 0: r2 == 0 pairs contribute nothing
    _check_pass(NB, oracle, pos, vel, mass, theta=0.5, eps=0.0)


@pytest.mark.parametrize("scale,offset,eps", [(1e3, 5e3, 1.0), (1e-6, 2e-6, 1e-9), (1e6, -3e6, 1e3),
                                              (1.0, 0.0, 1e-3)])
def test_translated_and_scaled_inputs(NB, oracle, scale, offset, eps):
    """The fp32 filters' error bounds carry the coordinate range R (DESIGN.md
    "fp32 filter", "T filter"): translated, small and large coordinates must
    still give exactly the oracle's keys, trees and interaction lists
    (undecided cases fall back to the fp64 test).  The scales keep the fp32
    interaction's intermediate m (r^2 + eps^2)^(-3/2) inside the fp32 range
    (the documented limit of the fp32 mode, [A15]; at 1e-12 it overflows)."""
    pos, vel, mass = generate("disks", 12_007, 12)
    pos = (pos.astype(np.float64) * scale + offset).astype(np.float32)
    _check_pass(NB, oracle, pos, vel, mass, theta=0.5, eps=eps)


def test_far_offset_keeps_the_lists(NB, oracle):
    """Coordinates 10^4 times the system size away from the origin: the fp32
    state then resolves the near field only to ~1e-3 of a body spacing, so
    fp32 monopoles (c32) may differ from the oracle's fp64 ones beyond the
    force tolerance, but every opening decision -- hence every list and
    count -- is still the oracle's (the filters widen with R)."""
    pos, vel, mass = generate("disks", 12_007, 14)
    pos = (pos.astype(np.float64) + 1e4).astype(np.float32)
    sim = _run_gpu(NB, pos, vel, mass, 0.5, 16)
    ref = oracle.step(pos, vel, mass, theta=0.5, eps=EPS, dt=DT, key_bits=16, integrate=False)
    assert (sim.debug_keys() == ref.keys).all() and (sim.debug_perm() == ref.perm).all()
    assert (sim.get_interactions()[ref.ids] == ref.count).all()


@pytest.mark.parametrize("theta", [1.2, 4.0])
def test_wide_opening_angles(NB, oracle, theta):
    """theta beyond 1/sqrt(3): an accepted node may contain the target [A4]
    (no special case on either side); lists and counts still equal."""
    pos, vel, mass = generate("plummer", 9_001, 13)
    _check_pass(NB, oracle, pos, vel, mass, theta=theta)


def test_dominant_central_mass(NB, oracle):
    """A galaxy with a central mass 10^6 times the others (node COMs pulled
    onto one body, masses spanning 6 decades in the fp64 moments and the
    fp32 records): records bit-exact, lists equal, accelerations in tolerance."""
    pos, vel, mass = generate("plummer", 10_001, 15)
    pos[0] = 0.0
    mass = mass.copy()
    mass[0] = mass[1] * 1e6
    _check_pass(NB, oracle, pos, vel, mass, theta=0.5)


def test_mixed_masses(NB, oracle):
    pos, vel, _ = generate("clustered", 8000, 9)
    mass = np.random.default_rng(9).lognormal(0.0, 1.0, 8000).astype(np.float32)
    _check_pass(NB, oracle, pos, vel, mass, theta=0.6)


def test_traversal_variants_agree(NB, oracle):
    pos, vel, mass = generate("disks", 20_000, 10)
    s0 = _run_gpu(NB, pos, vel, mass, 0.5, 16, traversal=0)
    s1 = _run_gpu(NB, pos, vel, mass, 0.5, 16, traversal=1)
    assert (s0.get_interactions() == s1.get_interactions()).all()
    e = rel_errors(s0.get_accel(), s1.get_accel())
    assert e.max() < 1e-5


@pytest.mark.parametrize("name,n,seed,theta", [("plummer", 9_001, 3, 0.5), ("clustered", 12_000, 4, 0.8),
                                                ("uniform", 1, 1, 0.5), ("uniform", 37, 2, 0.0)])
def test_paper_skiplist_variant_parity(NB, oracle, name, n, seed, theta):
    """Traversal variant 2 (the paper's per-body stackless skip-list DFS,
    P:222/P:245) against the oracle: counts equal, accelerations in
    tolerance, and the same lists as the default variant."""
    pos, vel, mass = generate(name, n, seed)
    _check_pass(NB, oracle, pos, vel, mass, theta=theta, levels=False, traversal=2)
    s0 = _run_gpu(NB, pos, vel, mass, theta, 16, traversal=0)
    s2 = _run_gpu(NB, pos, vel, mass, theta, 16, traversal=2)
    assert (s0.get_interactions() == s2.get_interactions()).all()


def test_paper_skiplist_variant_steps(NB):
    """Variant 2 inside whole steps (graph capture) matches the default."""
    pos, vel, mass = generate("disks", 20_000, 11)
    out = []
    for v in (0, 2):
        sim = NB(len(pos), 0.5, EPS, DT, key_bits=16, traversal=v)
        sim.set_bodies(pos, vel, mass)
        sim.step(3)
        out.append((sim.get_positions(), sim.get_interactions()))
    assert (out[0][1] == out[1][1]).all()
    assert rel_errors(out[0][0], out[1][0]).max() < 1e-5


def test_step_parity_and_determinism(NB, oracle):
    """One full step (force + leapfrog) against the oracle; two GPU runs are
    bit-identical (no float atomics anywhere); graph == plain launches."""
    pos, vel, mass = generate("plummer", 50_000, 11)
    outs = []
    for graph in (True, False, True):
        sim = NB(len(pos), 0.5, EPS, DT, key_bits=16, use_graph=graph)
        sim.set_bodies(pos, vel, mass)
        sim.step(1)
        outs.append((sim.get_positions(), sim.get_velocities(), sim.get_accel()))
    for o in outs[1:]:
        for a, b in zip(outs[0], o):
            assert (a == b).all()
    ref = oracle.step(pos, vel, mass, theta=0.5, eps=EPS, dt=DT, key_bits=16)
    x_gpu, v_gpu, a_gpu = outs[0]
    order = ref.ids
    assert_acc_close(a_gpu[order], ref.acc)
    # v = v0 + a dt; positions move by v dt: differences are a-rounding sized
    dv = np.abs(v_gpu[order].astype(float) - ref.vel.astype(float)).max()
    assert dv <= 1e-2 * DT * np.abs(ref.acc).max() + 1e-6 * np.abs(ref.vel).max()
    dx = np.abs(x_gpu[order].astype(float) - ref.pos.astype(float)).max()
    assert dx <= 2 * np.spacing(np.abs(ref.pos).max().astype(np.float32)) + DT * dv


def test_ten_steps_track_the_oracle(NB, oracle):
    """10 steps (config 2's loop, small N): trajectories stay within the
    drift the tolerances allow."""
    n, steps = 20_000, 10
    pos, vel, mass = generate("plummer", n, 12)
    sim = NB(n, 0.5, EPS, DT, key_bits=16)
    sim.set_bodies(pos, vel, mass)
    sim.step(steps)
    xg = sim.get_positions()
    x, v, m, ids = pos, vel, mass, np.arange(n)
    amax = 0.0
    for _ in range(steps):
        r = oracle.step(x, v, m, ids, theta=0.5, eps=EPS, dt=DT, key_bits=16)
        x, v, m, ids = r.pos, r.vel, r.mass, r.ids
        amax = max(amax, float(np.abs(r.acc).max()))
    xo = np.empty_like(x)
    xo[ids] = x
    # |dx| <= steps^2 dt^2 max|da| with |da| <= 1e-2 |a| per body and step,
    # plus fp32 rounding of the positions each step
    bound = steps * steps * DT * DT * 1e-2 * amax + steps * 2 * np.spacing(np.float32(np.abs(x).max()))
    assert np.abs(xg.astype(float) - xo.astype(float)).max() <= bound
    st = sim.stats()
    assert st["steps"] == steps and st["interactions"] > 0


def test_device_pointers_round_trip(NB):
    import torch
    pos, vel, mass = generate("uniform", 5000, 13)
    tp, tv, tm = (torch.from_numpy(a).cuda() for a in (pos, vel, mass))
    sim = NB(5000, 0.5, EPS, DT)
    sim.set_bodies(tp, tv, tm)
    out = torch.empty((5000, 3), dtype=torch.float32, device="cuda")
    sim.get_positions(out)
    assert (out.cpu().numpy() == pos).all()
    sim.compute_accel()
    a_host = sim.get_accel()
    sim.get_accel(out)
    assert (out.cpu().numpy() == a_host).all()


def test_invalid_bodies_rejected(NB):
    from paper_conf_sc_casselldahg24_b200 import NBodyError
    pos, vel, mass = generate("uniform", 100, 14)
    sim = NB(100, 0.5, EPS, DT)
    bad = mass.copy()
    bad[5] = 0.0
    with pytest.raises(NBodyError):
        sim.set_bodies(pos, vel, bad)
    pos2 = pos.copy()
    pos2[3, 1] = np.nan
    with pytest.raises(NBodyError):
        sim.set_bodies(pos2, vel, mass)
    with pytest.raises(NBodyError):
        sim.step(1)  # nothing loaded
    sim.set_bodies(pos, vel, mass)
    sim.step(1)


# ---------------------------------------------------------------- full size --
def _sampled_full_size(NB, oracle, name, n, seed, nsample, theta=0.5):
    pos, vel, mass = generate(name, n, seed)
    sim = NB(n, theta, EPS, DT, key_bits=16)
    sim.set_bodies(pos, vel, mass)
    sim.compute_accel()
    rng = np.random.default_rng(seed)
    targets = np.sort(rng.choice(n, nsample, replace=False))
    ref = oracle.step(pos, vel, mass, theta=theta, eps=EPS, dt=DT, key_bits=16, integrate=False, targets=targets)
    assert (sim.debug_keys() == ref.keys).all()
    assert (sim.debug_perm() == ref.perm).all()
    # node records: the top 8 levels entirely, sampled nodes below
    for l in range(1, ref.tree.L + 1):
        pred, rec, box = sim.debug_level(l)
        d = ref.tree.level(l)
        sel = slice(None) if len(pred) <= 4096 else rng.choice(len(pred), 4096, replace=False)
        assert (pred[sel, :3] == d.com[sel]).all() and (pred[sel, 3] == d.s2[sel]).all()
        assert (rec[sel, :3] == d.c32[sel]).all() and (rec[sel, 3] == d.m32[sel]).all()
    acc = sim.get_accel()
    cnt = sim.get_interactions()
    ids_t = ref.ids[targets]
    assert (cnt[ids_t] == ref.count).all()
    assert_acc_close(acc[ids_t], ref.acc)


def test_config2_plummer_1M_sampled(NB, oracle):
    _sampled_full_size(NB, oracle, "plummer", 1_000_000, 2, 3000)


@pytest.mark.slow
def test_config3_disks_10M_sampled(NB, oracle):
    _sampled_full_size(NB, oracle, "disks", 10_000_000, 3, 2000)


@pytest.mark.slow
@pytest.mark.parametrize("name,seed,theta", [("uniform", 5, 0.3), ("clustered", 6, 0.8)])
def test_config5_theta_sweep_10M_sampled(NB, oracle, name, seed, theta):
    """Config 5 (theta sweep at N = 10^7, uniform vs clustered) at its two
    extremes: the narrowest opening angle on the uniform cube (longest lists)
    and the widest on the clustered set (accepted nodes may contain the
    target, [A4]); keys, permutation, node records, counts and sampled
    accelerations against the oracle."""
    _sampled_full_size(NB, oracle, name, 10_000_000, seed, 1000, theta=theta)


@pytest.mark.slow
def test_config3_bench_launch_configuration(NB, oracle):
    """Config 3 at full size in the configuration bench.py times: nbody_step
    replayed from its CUDA graph on a caller (torch) stream.  The second
    step's force pass runs on the state left by the first (slot order and
    all), which is read back with nbody_get_state and given to the oracle;
    the counts and accelerations of sampled bodies must match it."""
    import torch
    n = 10_000_000
    pos, vel, mass = generate("disks", n, 3)
    stream = torch.cuda.Stream()
    sim = NB(n, 0.5, EPS, DT, key_bits=16, stream=stream.cuda_stream)
    sim.set_bodies(pos, vel, mass)
    sim.step(1)
    pm, vi = sim.get_state()              # slot order after step 1
    ids_state = vi[:, 3].view(np.int32).copy()
    sim.step(1)                           # its force pass runs on that state
    acc = sim.get_accel()
    cnt = sim.get_interactions()
    targets = np.sort(np.random.default_rng(33).choice(n, 1500, replace=False))
    ref = oracle.step(pm[:, :3], vi[:, :3], pm[:, 3], ids_state, theta=0.5, eps=EPS, dt=DT, key_bits=16,
                      integrate=False, targets=targets)
    ids_t = ref.ids[targets]
    assert (cnt[ids_t] == ref.count).all()
    assert_acc_close(acc[ids_t], ref.acc)


# ------------------------------------------------------- NEXT-1 all-pairs --
@pytest.mark.parametrize("name,n,seed,eps", [("plummer", 5000, 60, 1e-3), ("uniform", 3001, 61, 0.0)])
def test_direct_accel_matches_oracle_direct_sum(NB, oracle, name, n, seed, eps):
    """The GPU all-pairs kernel (fp64) equals the oracle's direct sum D to
    fp64 rounding (different summation order only)."""
    pos, vel, mass = generate(name, n, seed)
    sim = NB(n, 0.5, eps, DT)
    sim.set_bodies(pos, vel, mass)
    ids = np.random.default_rng(seed).choice(n, 257, replace=False)
    got = sim.direct_accel(ids)
    ref = oracle.direct(pos, mass, eps, targets=ids)
    assert rel_errors(got, ref).max() <= 1e-12


def test_direct_accel_at_10M_sampled(NB, oracle):
    n = 10_000_000
    pos, vel, mass = generate("disks", n, 3)
    sim = NB(n, 0.5, EPS, DT)
    sim.set_bodies(pos, vel, mass)
    ids = np.random.default_rng(3).choice(n, 48, replace=False)
    got = sim.direct_accel(ids)
    ref = oracle.direct(pos, mass, EPS, targets=ids)
    assert rel_errors(got, ref).max() <= 1e-11
    # Barnes-Hut at theta = 0.5 against the exact field: accuracy is reported
    # by the theta sweep; here only a sanity bound
    sim.compute_accel()
    bh = sim.get_accel()[ids]
    assert np.median(rel_errors(bh, got)) < 1e-2


@pytest.mark.parametrize("n", [1000, 1025, 70_001, 2_000_003])
def test_build_variants_bit_identical(NB, n):
    """Fused-subtree build == level-by-level build, every level."""
    pos, vel, mass = generate("clustered", n, 70)
    sims = []
    for variant in (0, 1):
        s = NB(n, 0.5, EPS, DT)
        s.set_option(6, variant)  # NBODY_OPT_BUILD
        s.set_bodies(pos, vel, mass)
        s.compute_accel()
        sims.append(s)
    L = sims[0].stats()["levels"]
    for l in range(1, L + 1):
        for a, b in zip(sims[0].debug_level(l), sims[1].debug_level(l)):
            assert (a == b).all(), l
    assert (sims[0].get_accel() == sims[1].get_accel()).all()


# ------------------------------------------------- NEXT-3(iii) tree reuse ---
def test_tree_reuse_step_is_a_refit(NB):
    """With dt = 0 a reuse step keeps the order and positions, so it must give
    exactly the accelerations of a fresh pass."""
    n = 40_000
    pos, vel, mass = generate("clustered", n, 83)
    s = NB(n, 0.5, EPS, 0.0, use_graph=True)
    s.set_option(7, 3)  # NBODY_OPT_SORT_EVERY
    s.set_bodies(pos, vel, mass)
    s.step(1)
    pm0, vi0 = s.get_state()
    a0 = s.get_accel()
    s.step(1)  # reuse step
    pm1, vi1 = s.get_state()
    assert (vi1[:, 3].view(np.int32) == vi0[:, 3].view(np.int32)).all()
    assert (s.get_accel() == a0).all()


def test_tree_reuse_against_oracle(NB, oracle):
    """NEXT-3(iii) [A23] on identical inputs: the reuse step's force pass runs
    on the state the sorting step left (read back with nbody_get_state), and
    the oracle's resort=False step is given exactly that state, so the trees
    and every interaction list must be identical: counts equal for every
    body, accelerations within the north-star tolerances, and the update
    within its rounding bound."""
    n, dt = 30_000, 1e-3
    for name, seed, theta in (("plummer", 84, 0.5), ("disks", 85, 0.8)):
        pos, vel, mass = generate(name, n, seed)
        s = NB(n, theta, EPS, dt)
        s.set_option(7, 2)
        s.set_bodies(pos, vel, mass)
        s.step(1)
        pm, vi = s.get_state()                 # slot order and state after the sorting step
        ids0 = vi[:, 3].view(np.int32).copy()
        s.step(1)                              # reuse: same slot order, tree refitted at the new positions
        pm1, vi1 = s.get_state()
        assert (vi1[:, 3].view(np.int32) == ids0).all()
        r1 = oracle.step(pm[:, :3], vi[:, :3], pm[:, 3], ids0, theta=theta, eps=EPS, dt=dt, resort=False)
        assert (r1.ids == ids0).all()
        cnt = s.get_interactions()[r1.ids]
        assert (cnt == r1.count).all(), f"{name}: {int((cnt != r1.count).sum())} bodies with other lists"
        assert_acc_close(s.get_accel()[r1.ids], r1.acc)
        _check_update(pm1[:, :3], vi1[:, :3], r1, dt)


def test_tree_reuse_with_quadrupoles_against_oracle(NB, oracle):
    """NEXT-3(iii) with NEXT-4 [A23][A24]: a reuse step refits the second
    moments too; on the reuse step's input state the oracle's
    resort=False, quad=True step has the same lists and moments."""
    n, dt = 20_000, 1e-3
    pos, vel, mass = generate("clustered", n, 86)
    s = NB(n, 0.6, EPS, dt, multipole=2)
    s.set_option(7, 2)
    s.set_bodies(pos, vel, mass)
    s.step(1)
    pm, vi = s.get_state()
    ids0 = vi[:, 3].view(np.int32).copy()
    s.step(1)  # reuse step
    r1 = oracle.step(pm[:, :3], vi[:, :3], pm[:, 3], ids0, theta=0.6, eps=EPS, dt=dt, resort=False, quad=True)
    assert (r1.ids == ids0).all()
    assert (s.get_interactions()[r1.ids] == r1.count).all()
    assert_acc_close(s.get_accel()[r1.ids], r1.acc)


def _check_update(x_gpu, v_gpu, ref, dt=DT):
    """Leapfrog O8 on the same input: v = v0 + a dt, x = x0 + v dt with the
    GPU's fp32 a (within the acceleration tolerance) -- differences are
    acceleration-error and fp32-rounding sized.  x_gpu, v_gpu in the oracle's
    sorted slot order."""
    dv = np.abs(v_gpu.astype(float) - ref.vel.astype(float)).max()
    assert dv <= 1e-2 * dt * np.abs(ref.acc).max() + 1e-6 * np.abs(ref.vel).max() + 1e-30
    dx = np.abs(x_gpu.astype(float) - ref.pos.astype(float)).max()
    assert dx <= 2 * np.spacing(np.abs(ref.pos).max().astype(np.float32)) + dt * dv


# --------------------------------------------------- NEXT-4 quadrupoles ------
@pytest.mark.parametrize("name,n,seed,theta", [("plummer", 20_000, 93, 0.5), ("disks", 30_001, 94, 0.8),
                                               ("clustered", 1025, 95, 0.6), ("uniform", 3, 96, 0.5)])
def test_quadrupole_parity(NB, oracle, name, n, seed, theta):
    pos, vel, mass = generate(name, n, seed)
    sim = NB(n, theta, EPS, DT, multipole=2)
    sim.set_bodies(pos, vel, mass)
    sim.compute_accel()
    ref = oracle.step(pos, vel, mass, theta=theta, eps=EPS, dt=DT, integrate=False, quad=True)
    for l in range(1, ref.tree.L + 1):  # second moments bit-exact [A24]
        assert (sim.debug_quad(l) == ref.tree.level_quad(l)).all(), l
    assert (sim.get_interactions()[ref.ids] == ref.count).all()
    assert_acc_close(sim.get_accel()[ref.ids], ref.acc)
    v1 = NB(n, theta, EPS, DT, multipole=2, traversal=1)  # mask-walk variant
    v1.set_bodies(pos, vel, mass)
    v1.compute_accel()
    assert (v1.get_interactions() == sim.get_interactions()).all()
    assert rel_errors(v1.get_accel(), sim.get_accel()).max() < 1e-4


def test_quadrupole_is_more_accurate_at_1M(NB):
    n = 1_000_000
    pos, vel, mass = generate("plummer", n, 2)
    ids = np.random.default_rng(97).choice(n, 500, replace=False)
    errs = {}
    for mp in (1, 2):
        sim = NB(n, 0.5, EPS, DT, multipole=mp)
        sim.set_bodies(pos, vel, mass)
        sim.compute_accel()
        exact = sim.direct_accel(ids)
        errs[mp] = float(np.sqrt(np.mean(rel_errors(sim.get_accel()[ids], exact) ** 2)))
    assert errs[2] < 0.5 * errs[1], errs
