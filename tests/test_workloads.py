"""Seeded generators: determinism, chunk keying and distribution statistics."""
import math

import numpy as np
import pytest

from workloads import generate
from workloads import generators as G


@pytest.mark.parametrize("name", G.NAMES)
def test_deterministic_and_typed(name):
    a = generate(name, 5000, 7)
    b = generate(name, 5000, 7)
    for x, y in zip(a, b):
        assert x.dtype == np.float32 and (x == y).all()
    assert a[0].shape == (5000, 3) and a[1].shape == (5000, 3) and a[2].shape == (5000,)
    assert np.isfinite(a[0]).all() and np.isfinite(a[1]).all()
    assert (a[2] == np.float32(1 / 5000)).all()


def test_chunk_keying_is_prefix_stable(monkeypatch):
    monkeypatch.setattr(G, "CHUNK", 1000)
    a = generate("uniform", 3500, 3)[0]
    b = generate("uniform", 2500, 3)[0]
    assert (a[:2000] == b[:2000]).all()  # whole chunks do not depend on N


def test_plummer_half_mass_radius():
    pos, vel, _ = generate("plummer", 200_000, 2)
    r = np.linalg.norm(pos.astype(float), axis=1)
    a = 3 * math.pi / 16
    # half-mass radius of a Plummer sphere: a / sqrt(2^(2/3) - 1) (0.999 cut-off shifts it by < 0.1%)
    assert np.median(r) == pytest.approx(a / math.sqrt(2 ** (2 / 3) - 1), rel=0.01)
    # virial (Henon) units: E = -1/4, so T = 1/4 and 2T/|W| = 1 (|W| = 1/2)
    t = 0.5 * (vel.astype(float) ** 2).sum(axis=1).mean()
    assert t == pytest.approx(0.25, rel=0.03)


def test_two_disks_geometry():
    n = 100_000
    pos, vel, _ = generate("disks", n, 3)
    d1, d2 = pos[: n // 2].astype(float), pos[n // 2:].astype(float)
    assert np.allclose(d1.mean(axis=0), [-4, -1, 0], atol=0.05)
    assert np.allclose(d2.mean(axis=0), [4, 1, 0], atol=0.05)
    assert np.allclose(vel[: n // 2].mean(axis=0), [0.3, 0, 0], atol=0.01)
    assert np.allclose(vel[n // 2:].mean(axis=0), [-0.3, 0, 0], atol=0.01)
    assert d1[:, 2].std() == pytest.approx(0.05, rel=0.03)  # thin, untilted
    assert d2[:, 2].std() > 0.5  # tilted by 0.5 rad about x
    r = np.linalg.norm(d1[:, :2] - [-4, -1], axis=1)
    assert r.max() <= 5.0 + 1e-5 and r.mean() == pytest.approx(1.83, rel=0.02)  # Gamma(2,1) truncated at 5


def test_clustered_has_64_clusters():
    n = 64 * 500
    pos, _, _ = generate("clustered", n, 4)
    centres, _ = G._cluster_params(4)
    for c in range(0, 64, 9):
        blk = pos[c * 500:(c + 1) * 500].astype(float)
        assert np.linalg.norm(np.median(blk, axis=0) - centres[c]) < 0.03
