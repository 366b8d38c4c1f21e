"""Seeded synthetic workloads for the AFMM near-field P2P path.

This module is the ONE piece shared by the oracle side (``oracle/``, ``tests/``)
and the product side (``bench.py``, ``__graft_entry__``).  It draws body
positions and masses only; it contains none of the method's arithmetic (no tree,
no U-list, no interaction law).

Workloads follow the paper's test problems:
  * "gravitational problem ... Every particle in this system has a mass of
    1.0kg" -- PAPER.md L22 SVIII.B.  We use m_i = 1/N (a pure scale change, see
    DESIGN.md reading R19).
  * "ten million particles distributed in a Plummer distribution" -- L22 SVIII.C/D.
  * "colliding galaxies" -- L10 Abstract; dynamic workload "initially contained
    within 1/64 th of the simulation space" -- L24 SIX.A.
  * uniform cube -- BASELINE.json configs[0].

Randomness is a counter-based splitmix64: draw k of stream ``s`` under seed
``seed`` is ``mix(seed_key(seed, s) + (k+1)*GOLDEN)``; u = (r >> 11) * 2^-53 in
[0, 1).  Positions are generated in fp64 and rounded once to fp32 (RN); both the
oracle and the CUDA path consume those fp32 values.
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
PLUMMER_RMAX = 10.0          # truncation radius (reading R20)
PLUMMER_ATTEMPTS = 8         # rejection attempts per body before clamping to RMAX


def _mix(z: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def _seed_key(seed: int, stream: int) -> np.uint64:
    with np.errstate(over="ignore"):
        s = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) * GOLDEN + np.uint64(stream & 0xFFFFFFFF)
        return _mix(np.array([s], dtype=np.uint64))[0]


def uniform01(seed: int, stream: int, k: np.ndarray) -> np.ndarray:
    """u_k in [0,1) (fp64) for counter array ``k`` of stream ``stream``."""
    key = _seed_key(seed, stream)
    with np.errstate(over="ignore"):
        z = key + (k.astype(np.uint64) + np.uint64(1)) * GOLDEN
    r = _mix(z)
    return (r >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def _as_f32_bodies(pos: np.ndarray, n: int):
    x = pos[:, 0].astype(np.float32)
    y = pos[:, 1].astype(np.float32)
    z = pos[:, 2].astype(np.float32)
    m = np.full(n, np.float32(1.0 / n), dtype=np.float32)
    return x, y, z, m


def uniform_cube(n: int, seed: int):
    """n bodies uniform in [0,1)^3 (BASELINE.json configs[0])."""
    k = np.arange(n, dtype=np.uint64)
    pos = np.empty((n, 3), dtype=np.float64)
    for c in range(3):
        pos[:, c] = uniform01(seed, 1, k * np.uint64(3) + np.uint64(c))
    return _as_f32_bodies(pos, n)


def _plummer_positions(n: int, seed: int, stream: int) -> np.ndarray:
    """Plummer sphere, scale a=1 (Aarseth-Henon-Wielen inverse-CDF sampling).

    r = (X^(-2/3) - 1)^(-1/2), X in (0,1]; resampled while r > RMAX (up to
    PLUMMER_ATTEMPTS attempts, then clamped); isotropic direction.
    Draw index for body i, attempt a, component c: (i*PLUMMER_ATTEMPTS + a)*4 + c.
    """
    idx = np.arange(n, dtype=np.uint64)
    r = np.full(n, np.inf)
    done = np.zeros(n, dtype=bool)
    ct = np.zeros(n)
    ph = np.zeros(n)
    for a in range(PLUMMER_ATTEMPTS):
        todo = np.nonzero(~done)[0]
        if todo.size == 0:
            break
        base = (idx[todo] * np.uint64(PLUMMER_ATTEMPTS) + np.uint64(a)) * np.uint64(4)
        X = 1.0 - uniform01(seed, stream, base)          # (0, 1]
        with np.errstate(divide="ignore"):
            rr = 1.0 / np.sqrt(X ** (-2.0 / 3.0) - 1.0)
        ok = rr <= PLUMMER_RMAX
        acc = todo[ok]
        r[acc] = rr[ok]
        ct[acc] = 2.0 * uniform01(seed, stream, base[ok] + np.uint64(1)) - 1.0
        ph[acc] = 2.0 * np.pi * uniform01(seed, stream, base[ok] + np.uint64(2))
        done[acc] = True
    rest = np.nonzero(~done)[0]
    if rest.size:
        base = (idx[rest] * np.uint64(PLUMMER_ATTEMPTS)) * np.uint64(4)
        r[rest] = PLUMMER_RMAX
        ct[rest] = 2.0 * uniform01(seed, stream, base + np.uint64(1)) - 1.0
        ph[rest] = 2.0 * np.pi * uniform01(seed, stream, base + np.uint64(2))
    st = np.sqrt(np.maximum(0.0, 1.0 - ct * ct))
    pos = np.empty((n, 3))
    pos[:, 0] = r * st * np.cos(ph)
    pos[:, 1] = r * st * np.sin(ph)
    pos[:, 2] = r * ct
    return pos


def plummer(n: int, seed: int):
    """n-body Plummer sphere (a = 1, r <= 10), centred at the origin."""
    return _as_f32_bodies(_plummer_positions(n, seed, 2), n)


COLLIDE_CENTRES = ((-5.0, -1.0, 0.0), (5.0, 1.0, 0.0))


def colliding(n: int, seed: int):
    """Two Plummer spheres of n/2 (and n - n/2) bodies centred at (-5,-1,0), (+5,+1,0)."""
    na = n // 2
    pa = _plummer_positions(na, seed, 3) + np.array(COLLIDE_CENTRES[0])
    pb = _plummer_positions(n - na, seed, 4) + np.array(COLLIDE_CENTRES[1])
    return _as_f32_bodies(np.concatenate([pa, pb]), n)


def _plummer_velocities(pos: np.ndarray, mass: float, seed: int, stream: int) -> np.ndarray:
    """Isotropic Plummer velocities (a = 1, G = 1, sphere mass `mass`): speed
    v = q * v_esc(r), v_esc = sqrt(2 mass) (1 + r^2)^(-1/4), q drawn by rejection
    from g(q) = q^2 (1 - q^2)^(7/2) (Aarseth-Henon-Wielen).  Draw index for body
    i, attempt a, component c: (i*64 + a)*4 + c."""
    n = pos.shape[0]
    idx = np.arange(n, dtype=np.uint64)
    q = np.full(n, 0.5)
    done = np.zeros(n, dtype=bool)
    for a in range(64):
        todo = np.nonzero(~done)[0]
        if todo.size == 0:
            break
        base = (idx[todo] * np.uint64(64) + np.uint64(a)) * np.uint64(4)
        qq = uniform01(seed, stream, base)
        gg = 0.1 * uniform01(seed, stream, base + np.uint64(1))
        ok = gg < qq * qq * (1.0 - qq * qq) ** 3.5
        q[todo[ok]] = qq[ok]
        done[todo[ok]] = True
    base = idx * np.uint64(64 * 4) + np.uint64(64 * 4 - 2)      # direction draws (disjoint indices)
    ct = 2.0 * uniform01(seed, stream + 100, base) - 1.0
    ph = 2.0 * np.pi * uniform01(seed, stream + 100, base + np.uint64(1))
    r2 = (pos ** 2).sum(1)
    v = q * np.sqrt(2.0 * mass) * (1.0 + r2) ** -0.25
    st = np.sqrt(np.maximum(0.0, 1.0 - ct * ct))
    return np.stack([v * st * np.cos(ph), v * st * np.sin(ph), v * ct], 1)


COLLIDE_BULK = ((0.5, 0.0, 0.0), (-0.5, 0.0, 0.0))


def colliding_with_velocities(n: int, seed: int):
    """C5 initial state: the colliding pair of `colliding` plus velocities --
    bulk (+0.5, 0, 0) for the sphere at x = -5 and (-0.5, 0, 0) for the one at
    x = +5 (approach along x), plus isotropic Plummer internal velocities.
    Returns fp32 (x, y, z, m, vx, vy, vz)."""
    na = n // 2
    pa = _plummer_positions(na, seed, 3)
    pb = _plummer_positions(n - na, seed, 4)
    va = _plummer_velocities(pa, na / n, seed, 5) + np.array(COLLIDE_BULK[0])
    vb = _plummer_velocities(pb, (n - na) / n, seed, 6) + np.array(COLLIDE_BULK[1])
    pos = np.concatenate([pa + np.array(COLLIDE_CENTRES[0]), pb + np.array(COLLIDE_CENTRES[1])])
    vel = np.concatenate([va, vb])
    x, y, z, m = _as_f32_bodies(pos, n)
    return x, y, z, m, vel[:, 0].astype(np.float32), vel[:, 1].astype(np.float32), vel[:, 2].astype(np.float32)


def c5_domain(x, y, z):
    """Fixed C5 domain (reading R9, "initially contained within 1/64 th
    of the simulation space"): the initial power-of-two cube (lo, k) grown 4x per
    axis (side 2^(k+2)) and centred on the initial cube.  Returns (lo[3], k)."""
    P = np.stack([x, y, z], 1).astype(np.float64)
    lo = P.min(0)
    ext = (P.max(0) - lo).max()
    k = int(np.frexp(ext)[1]) if ext > 0 else 0
    side = 2.0 ** k
    return lo - 1.5 * side, k + 2


def lattice(M: int):
    """One body at each cell centre of an M^3 grid on [0,1)^3 (U-list closed-form pin)."""
    c = (np.arange(M, dtype=np.float64) + 0.5) / M
    gx, gy, gz = np.meshgrid(c, c, c, indexing="ij")
    pos = np.stack([gx.ravel(), gy.ravel(), gz.ravel()], axis=1)
    return _as_f32_bodies(pos, pos.shape[0])


GENERATORS = {"uniform": uniform_cube, "plummer": plummer, "colliding": colliding}

# BASELINE.json configs -> concrete synthetic inputs.
CONFIGS = {
    "C1": dict(dist="uniform", n=4096, S=64, seed=1, eps2=1e-6),
    "C2": dict(dist="plummer", n=1 << 20, S=128, seed=2, eps2=1e-6),   # S swept 32..512
    "C3": dict(dist="colliding", n=1 << 22, S=128, seed=3, eps2=1e-6),
    "C4": dict(dist="plummer", n=1 << 24, S=256, seed=4, eps2=1e-6),
    "C5": dict(dist="colliding", n=1 << 20, S=128, seed=5, eps2=1e-4),
}


def make(name_or_dist: str, n: int | None = None, seed: int | None = None):
    """Return fp32 (x, y, z, m) for a named config ("C1".."C5") or a distribution."""
    if name_or_dist in CONFIGS:
        c = CONFIGS[name_or_dist]
        return GENERATORS[c["dist"]](n if n is not None else c["n"],
                                     seed if seed is not None else c["seed"])
    return GENERATORS[name_or_dist](n, seed)


def uniform_with_forces(n: int, seed: int):
    """Stokeslet workload (PAPER L26 SIX.B: "ten million sources in a uniform
    distribution"): positions uniform in [0,1)^3, forces with independent
    components uniform in [-1, 1).  Returns fp32 (x, y, z, fx, fy, fz)."""
    x, y, z, _ = uniform_cube(n, seed)
    k = np.arange(n, dtype=np.uint64)
    f = [(2.0 * uniform01(seed, 7, k * np.uint64(3) + np.uint64(c)) - 1.0).astype(np.float32) for c in range(3)]
    return x, y, z, f[0], f[1], f[2]


CONFIGS["C6"] = dict(dist="stokeslet", n=10_000_000, S=128, seed=6, eps2=1e-6)
