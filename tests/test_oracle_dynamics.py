"""Pins for the oracle's C5 pieces (CPU only): Enforce_S (PAPER L20 SVI.A with
Collapse L18 SIV.B / PushDown L18 SIV.C) and the KDK leapfrog (reading R23).

Enforce_S is pinned by invariants that determine its result uniquely given
the previous tree: capacity (no leaf above S), Collapse (every internal node
holds >= S bodies), PushDown maximality (a node internal now but not before
holds > S), the hysteresis (an internal node holding exactly S was internal
before), plus hand-built cases.  The leapfrog is pinned by exact free motion
and by a two-body circular orbit (radius, period, energy)."""
import numpy as np
import pytest

import oracle
import synth


def _nodes(T):
    return {(int(l), int(p)): (int(e - b), bool(leaf)) for l, p, b, e, leaf in
            zip(T.node_level, T.node_prefix, T.node_b, T.node_e, T.node_is_leaf)}


def _check_enforce(prev, new, S):
    pn, nn = _nodes(prev), _nodes(new)
    for (l, p), (cnt, leaf) in nn.items():
        assert cnt > 0                                              # no empty nodes
        if leaf:
            assert cnt <= S or l == 21                              # PushDown: no leaf above S
        else:
            assert cnt >= S                                         # Collapse: internal holds >= S
            was_internal = (l, p) in pn and not pn[(l, p)][1]
            if cnt == S:
                assert was_internal                                 # hysteresis: only kept parents
            if not was_internal:
                assert cnt > S                                      # new parents from PushDown only
        if l > 0:
            parent = nn[(l - 1, p >> 3)]
            assert not parent[1]                                    # parents are internal
    # leaves tile [0, N) in Morton order
    assert new.leaf_start[0] == 0 and (new.leaf_start[1:] == new.leaf_start[:-1] + new.leaf_count[:-1]).all()
    assert new.leaf_start[-1] + new.leaf_count[-1] == new.n


def test_enforce_unchanged_positions_is_identity():
    x, y, z, m = synth.make("plummer", 20000, 3)
    dom = (np.array([-16.0, -16.0, -16.0]), 5)
    T = oracle.Tree(x, y, z, 32, domain=dom)
    xs, ys, zs = T.sorted_bodies(x, y, z)
    T2 = T.enforce(xs, ys, zs)
    assert np.array_equal(T2.perm, np.arange(20000))
    for a in ("leaf_start", "leaf_count", "leaf_level", "leaf_prefix", "u_off", "u_idx"):
        assert np.array_equal(getattr(T2, a), getattr(T, a))


def test_enforce_invariants_along_a_trajectory():
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(20000, 5)
    dom = synth.c5_domain(x, y, z)
    S = 24
    T = oracle.Tree(x, y, z, S, domain=dom)
    px, py, pz, vx, vy, vz = (a[T.perm] for a in (x, y, z, vx, vy, vz))
    for step in range(6):
        px, py, pz = oracle.drift(px, py, pz, vx, vy, vz, 0.4)
        T2 = T.enforce(px, py, pz)
        _check_enforce(T, T2, S)
        px, py, pz, vx, vy, vz = (a[T2.perm] for a in (px, py, pz, vx, vy, vz))
        T = T2
    # the U-list of an enforced tree is still the exact box adjacency (see test_oracle)
    from tests.test_oracle import _adjacent_boxes, _leaf_boxes
    A, w = _leaf_boxes(T)
    dense = np.zeros((T.L, T.L), bool)
    dense[np.repeat(np.arange(T.L), np.diff(T.u_off)), T.u_idx] = True
    assert np.array_equal(dense, _adjacent_boxes(A, w))


def test_enforce_hand_built_collapse_pushdown_hysteresis():
    """Unit cube, S = 4.  Octant 0 holds 5 bodies (split), octant 7 holds 2.
    Move one body from octant 0 to octant 7: octant 0 now holds exactly S = 4
    and stays a parent (Enforce_S collapses only parents with FEWER than S);
    a fresh build would make it a leaf.  Then move another: 3 < S collapses.
    Then fill octant 7 to 5 > S: it is pushed down."""
    def pts(list_):
        a = np.array(list_, np.float32)
        return a[:, 0].copy(), a[:, 1].copy(), a[:, 2].copy()
    base = [[0.05, 0.05, 0.05], [0.3, 0.05, 0.05], [0.05, 0.3, 0.05], [0.05, 0.05, 0.3], [0.3, 0.3, 0.3],
            [0.95, 0.95, 0.95], [0.7, 0.7, 0.7], [0.0, 0.0, 0.0], [0.999, 0.999, 0.999]]
    dom = (np.zeros(3), 0)
    x, y, z = pts(base)
    T = oracle.Tree(x, y, z, 4, domain=dom)       # octant 0: 6 bodies (incl. origin), octant 7: 3
    nodes = _nodes(T)
    assert not nodes[(1, 0)][1] and nodes[(1, 0)][0] == 6
    moved = list(base)
    moved[1] = [0.8, 0.8, 0.8]
    moved[2] = [0.85, 0.8, 0.8]                  # octant 0 -> 4 bodies, octant 7 -> 5
    x2, y2, z2 = (a[T.perm] for a in pts(moved))
    T2 = T.enforce(x2, y2, z2)
    n2 = _nodes(T2)
    assert n2[(1, 0)] == (4, False)              # exactly S: kept as a parent (hysteresis)
    assert n2[(1, 7)] == (5, False)              # 5 > S: pushed down
    assert oracle.Tree(x2, y2, z2, 4, domain=dom) is not None
    fresh = _nodes(oracle.Tree(*pts(moved), 4, domain=dom))
    assert fresh[(1, 0)] == (4, True)            # a fresh build makes it a leaf
    _check_enforce(T, T2, 4)
    moved[3] = [0.9, 0.7, 0.9]                   # octant 0 -> 3 < S: collapsed
    x3, y3, z3 = (a[T2.perm] for a in (np.array(moved, np.float32)[T.perm][:, 0],
                                         np.array(moved, np.float32)[T.perm][:, 1],
                                         np.array(moved, np.float32)[T.perm][:, 2]))
    T3 = T2.enforce(x3, y3, z3)
    n3 = _nodes(T3)
    assert n3[(1, 0)] == (3, True)
    _check_enforce(T2, T3, 4)


def test_leapfrog_free_motion_exact():
    rng = np.random.default_rng(1)
    x, y, z = (rng.random(1000).astype(np.float32) for _ in range(3))
    vx, vy, vz = (np.round(rng.standard_normal(1000) * 64).astype(np.float32) / 64 for _ in range(3))
    zero = np.zeros(1000, np.float32)
    wx, wy, wz = oracle.kick(vx, vy, vz, zero, zero, zero, 0.125)
    assert np.array_equal(wx, vx) and np.array_equal(wy, vy) and np.array_equal(wz, vz)
    px, py, pz = oracle.drift(x, y, z, vx, vy, vz, 0.0625)
    assert np.array_equal(px, (x.astype(np.float64) + 0.0625 * vx).astype(np.float32))


def test_leapfrog_two_body_circular_orbit():
    """Equal masses m at distance d on a circle: v = sqrt(G m / (2 d)), period
    T = 2 pi sqrt(d^3 / (2 G m)).  KDK with the oracle's P2P force keeps the
    radius and energy to O(dt^2) and returns to the start after one period."""
    m, d = 0.5, 1.0
    v = np.sqrt(m / (2 * d))
    x = np.array([-d / 2, d / 2], np.float32)
    y = np.zeros(2, np.float32)
    z = np.zeros(2, np.float32)
    vx = np.zeros(2, np.float32)
    vy = np.array([-v, v], np.float32)
    vz = np.zeros(2, np.float32)
    M = np.full(2, m, np.float32)
    period = 2 * np.pi * np.sqrt(d ** 3 / (2 * m))
    nsteps = 2000
    dt = period / nsteps
    ls, lc, uo, ui = np.array([0], np.int32), np.array([2], np.int32), np.array([0, 1]), np.array([0], np.int32)

    def acc(x, y, z):
        _, ax, ay, az = oracle.p2p(x, y, z, M, ls, lc, uo, ui, 1.0, 0.0)
        return ax, ay, az

    def energy(x, y, z, vx, vy, vz):
        r = np.sqrt((x[1] - x[0]) ** 2 + (y[1] - y[0]) ** 2 + (z[1] - z[0]) ** 2)
        return 0.5 * m * float((vx.astype(float) ** 2 + vy.astype(float) ** 2 + vz.astype(float) ** 2).sum()) - m * m / r

    E0 = energy(x, y, z, vx, vy, vz)
    ax, ay, az = acc(x, y, z)
    radii = []
    for _ in range(nsteps):
        vx, vy, vz = oracle.kick(vx, vy, vz, ax, ay, az, dt / 2)
        x, y, z = oracle.drift(x, y, z, vx, vy, vz, dt)
        ax, ay, az = acc(x, y, z)
        vx, vy, vz = oracle.kick(vx, vy, vz, ax, ay, az, dt / 2)
        radii.append(np.hypot(x[1] - x[0], y[1] - y[0]))
    assert np.max(np.abs(np.array(radii) - d)) < 1e-4
    assert abs(energy(x, y, z, vx, vy, vz) - E0) < 1e-5 * abs(E0)
    assert abs(x[0] + d / 2) < 2e-3 and abs(y[0]) < 2e-3       # back at the start after one period


def test_c5_initial_state():
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(40000, 5)
    n = 40000
    # bulk velocities: the two spheres approach along x
    assert vx[: n // 2].mean() == pytest.approx(0.5, abs=0.02)
    assert vx[n // 2:].mean() == pytest.approx(-0.5, abs=0.02)
    # Plummer virial ratio 2K/|W| ~ 1 for each sphere (internal motion only), W = -3 pi M^2 / 32 (a = 1)
    va = np.stack([vx[: n // 2] - 0.5, vy[: n // 2], vz[: n // 2]], 1).astype(float)
    K = 0.5 * (m[: n // 2].astype(float)[:, None] * va ** 2).sum()
    W = -3 * np.pi * 0.5 ** 2 / 32
    assert 2 * K / abs(W) == pytest.approx(1.0, abs=0.08)      # truncation at r <= 10 lowers |W| a little
    lo, k = synth.c5_domain(x, y, z)
    side = 2.0 ** k
    assert (x >= lo[0]).all() and (x < lo[0] + side).all()
