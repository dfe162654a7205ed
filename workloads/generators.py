"""Seeded synthetic workloads for the Hilbert-BVH Barnes-Hut step.

This module is shared by the oracle tests and by the CUDA path's tests and
bench.  It holds NONE of the method's arithmetic (no bounding box, keys,
sort, tree or force): it only draws initial conditions.

The paper's workload is "a deterministic collision between two neighboring
Galaxies ... double precision ... theta factor of 0.5" (PAPER.md P:266-272,
Sec. V-A); it gives no generator parameters, so the recipes below are our
readings (restated in DESIGN.md "Input recipe"):

* ``uniform``   W1: x ~ U[-1,1)^3, v = 0.
* ``plummer``   W2: Plummer sphere, G = M = 1, scale a = 3*pi/16 (virial
  units).  Aarseth-Henon-Wielen (1974) sampling: r = a / sqrt(X^(-2/3) - 1)
  with X ~ U(0, 0.999]; isotropic.  Speed q * v_esc, v_esc = sqrt(2 M)
  (r^2 + a^2)^(-1/4), q by von Neumann rejection of q^2 (1 - q^2)^(7/2).
* ``disks``     W3: two exponential disks (mass 1/2 each).  R ~ Gamma(2, 1)
  truncated at 5, phi ~ U[0, 2 pi), z ~ N(0, 0.05^2); circular speed
  sqrt(M_enc(R)/R), M_enc(R) = 0.5 (1 - (1 + R) e^-R).  Disk 2 is tilted
  0.5 rad about x.  Centres (-4,-1,0) / (+4,+1,0); bulk velocities
  (+0.3,0,0) / (-0.3,0,0), i.e. towards each other.
* ``clustered`` W4: K = 64 Plummer clusters (a = 0.05, mass 1/K each),
  centres ~ U[-1,1)^3, bulk velocities ~ N(0, 0.1^2) per component.

Every body has mass 1/N.  Values are drawn in float64 with numpy's PCG64
and cast once to float32, in chunks of ``CHUNK`` bodies whose streams are
keyed by (seed, chunk index), so body i depends only on (name, seed, N, i)
and generating 10^8 bodies needs bounded memory.
"""
from __future__ import annotations

import math

import numpy as np

CHUNK = 1 << 20
NAMES = ("uniform", "plummer", "disks", "clustered")
N_CLUSTERS = 64


def _rng(seed: int, *key: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(np.random.SeedSequence(entropy=seed, spawn_key=key)))


def _isotropic(rng: np.random.Generator, n: int) -> np.ndarray:
    z = rng.uniform(-1.0, 1.0, n)
    phi = rng.uniform(0.0, 2.0 * math.pi, n)
    s = np.sqrt(np.maximum(0.0, 1.0 - z * z))
    return np.stack([s * np.cos(phi), s * np.sin(phi), z], axis=1)


def _plummer(rng: np.random.Generator, n: int, a: float, mass: float):
    """Aarseth-Henon-Wielen Plummer sample: positions and velocities, float64."""
    x = rng.uniform(0.0, 1.0, n)
    x = 0.999 * (1.0 - x)  # X in (0, 0.999]
    r = a / np.sqrt(x ** (-2.0 / 3.0) - 1.0)
    pos = r[:, None] * _isotropic(rng, n)
    q = np.empty(n)
    filled = 0
    while filled < n:
        m = max(64, 2 * (n - filled) + 64)
        x4 = rng.uniform(0.0, 1.0, m)
        x5 = rng.uniform(0.0, 1.0, m)
        ok = x4[0.1 * x5 < x4 * x4 * (1.0 - x4 * x4) ** 3.5]
        take = min(len(ok), n - filled)
        q[filled:filled + take] = ok[:take]
        filled += take
    vesc = math.sqrt(2.0 * mass) * (r * r + a * a) ** -0.25
    vel = (q * vesc)[:, None] * _isotropic(rng, n)
    return pos, vel


def _chunk_uniform(rng, lo, hi, n, seed):
    k = hi - lo
    return rng.uniform(-1.0, 1.0, (k, 3)), np.zeros((k, 3))


def _chunk_plummer(rng, lo, hi, n, seed):
    return _plummer(rng, hi - lo, 3.0 * math.pi / 16.0, 1.0)


def _disk(rng, k):
    r = rng.gamma(2.0, 1.0, k)
    bad = r > 5.0
    while bad.any():
        r[bad] = rng.gamma(2.0, 1.0, int(bad.sum()))
        bad = r > 5.0
    r = np.maximum(r, 1e-12)
    phi = rng.uniform(0.0, 2.0 * math.pi, k)
    z = rng.normal(0.0, 0.05, k)
    pos = np.stack([r * np.cos(phi), r * np.sin(phi), z], axis=1)
    menc = 0.5 * (1.0 - (1.0 + r) * np.exp(-r))
    vc = np.sqrt(menc / r)
    vel = np.stack([-vc * np.sin(phi), vc * np.cos(phi), np.zeros(k)], axis=1)
    return pos, vel


def _chunk_disks(rng, lo, hi, n, seed):
    half = n // 2
    idx = np.arange(lo, hi)
    second = idx >= half
    pos, vel = _disk(rng, hi - lo)
    t = 0.5
    c, s = math.cos(t), math.sin(t)
    rot = np.array([[1.0, 0.0, 0.0], [0.0, c, -s], [0.0, s, c]])
    pos[second] = pos[second] @ rot.T
    vel[second] = vel[second] @ rot.T
    pos += np.where(second[:, None], [4.0, 1.0, 0.0], [-4.0, -1.0, 0.0])
    vel += np.where(second[:, None], [-0.3, 0.0, 0.0], [0.3, 0.0, 0.0])
    return pos, vel


def _cluster_params(seed: int):
    rng = _rng(seed, 1 << 30)
    centres = rng.uniform(-1.0, 1.0, (N_CLUSTERS, 3))
    bulk = rng.normal(0.0, 0.1, (N_CLUSTERS, 3))
    return centres, bulk


def _chunk_clustered(rng, lo, hi, n, seed):
    centres, bulk = _cluster_params(seed)
    idx = np.arange(lo, hi, dtype=np.int64)
    cl = (idx * N_CLUSTERS) // n
    pos, vel = _plummer(rng, hi - lo, 0.05, 1.0 / N_CLUSTERS)
    return pos + centres[cl], vel + bulk[cl]


_CHUNKERS = {
    "uniform": _chunk_uniform,
    "plummer": _chunk_plummer,
    "disks": _chunk_disks,
    "clustered": _chunk_clustered,
}


def generate(name: str, n: int, seed: int, dtype=np.float32):
    """Return (pos float32[n,3], vel float32[n,3], mass float32[n]).

    ``vel`` is read as v_{-1/2} by the leapfrog (reading A14).
    ``dtype=np.float64`` returns the same fp64 draws without the final cast
    (inputs of the FP64 mode, NEXT-2); mass is then 1/N in fp64.
    """
    dtype = np.dtype(dtype)
    if dtype not in (np.float32, np.float64):
        raise ValueError("dtype must be float32 or float64")
    if name not in _CHUNKERS:
        raise ValueError(f"unknown workload {name!r}; expected one of {NAMES}")
    n = int(n)
    if n < 1:
        raise ValueError("n must be >= 1")
    pos = np.empty((n, 3), dtype)
    vel = np.empty((n, 3), dtype)
    f = _CHUNKERS[name]
    for c, lo in enumerate(range(0, n, CHUNK)):
        hi = min(n, lo + CHUNK)
        p, v = f(_rng(seed, c), lo, hi, n, seed)
        pos[lo:hi] = p
        vel[lo:hi] = v
    mass = np.full(n, dtype.type(1.0 / n), dtype)
    return pos, vel, mass


# Config table: the BASELINE.json configs as concrete inputs.
CONFIGS = {
    "cfg1": dict(workload="uniform", n=1024, seed=1, theta=0.5, eps=1e-3, dt=1e-3, steps=1),
    "cfg2": dict(workload="plummer", n=1_000_000, seed=2, theta=0.5, eps=1e-3, dt=1e-3, steps=10),
    "cfg3": dict(workload="disks", n=10_000_000, seed=3, theta=0.5, eps=1e-3, dt=1e-3, steps=10),
    "cfg4": dict(workload="clustered", n=100_000_000, seed=4, theta=0.5, eps=1e-3, dt=1e-3, steps=10),
}
