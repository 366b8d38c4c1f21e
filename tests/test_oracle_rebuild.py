"""Pins for the oracle's FineGrainedOptimize primitive (CPU only): rebuild with
the previous structure kept and per-node Collapse / PushDown edits (PAPER L18
SIV.B "collapse", SIV.C "pushdown", L20 SVI.B; reading R27).

Independent checks: the octant of every body is recomputed here with numpy
from the fixed domain (floor((x - lo) 2^(21-k)), bit 20-l of each axis), so a
PushDown is checked against a brute-force split; a Collapse is checked against
the union of the twig's children; KEEP without motion is the identity; KEEP
after motion keeps every previous parent that still holds bodies and creates
no new parent."""
import numpy as np

import oracle
import synth

DOM = (np.array([-16.0, -16.0, -16.0]), 5)


def _leaves(T):
    return {(int(l), int(p)): int(c) for l, p, c in zip(T.leaf_level, T.leaf_prefix, T.leaf_count)}


def _internal(T):
    return {(int(l), int(p)) for l, p, leaf in zip(T.node_level, T.node_prefix, T.node_is_leaf) if not leaf}


def _q(v, lo, k):
    return np.clip(np.floor((v.astype(np.float64) - lo) * 2.0 ** (21 - k)), 0, 2 ** 21 - 1).astype(np.int64)


def _tree():
    x, y, z, m = synth.make("plummer", 12000, 7)
    T = oracle.Tree(x, y, z, 24, domain=DOM)
    return T, T.sorted_bodies(x, y, z)


def _valid(T):
    assert T.leaf_start[0] == 0 and (T.leaf_start[1:] == T.leaf_start[:-1] + T.leaf_count[:-1]).all()
    assert int(T.leaf_count.sum()) == T.n and (T.leaf_count > 0).all()


def test_keep_without_motion_is_identity():
    T, (xs, ys, zs) = _tree()
    T2 = T.rebuild(xs, ys, zs, mode=2)
    assert np.array_equal(T2.perm, np.arange(T.n))
    for a in ("leaf_start", "leaf_count", "leaf_level", "leaf_prefix", "u_off", "u_idx", "node_prefix"):
        assert np.array_equal(getattr(T2, a), getattr(T, a))


def test_collapse_twigs_merges_their_children():
    T, (xs, ys, zs) = _tree()
    leaves, internal = _leaves(T), _internal(T)
    kids = {}
    for (l, p), c in leaves.items():
        kids.setdefault((l - 1, p >> 3), []).append(((l, p), c))
    nchild = {}
    for l, p in zip(T.node_level, T.node_prefix):
        if l > 0:
            nchild[(int(l) - 1, int(p) >> 3)] = nchild.get((int(l) - 1, int(p) >> 3), 0) + 1
    twigs = sorted(k for k in internal if k in kids and len(kids[k]) == nchild[k])[:7]
    assert len(twigs) == 7
    T2 = T.rebuild(xs, ys, zs, mode=2, edits=[(l, p, 1) for l, p in twigs])
    _valid(T2)
    want = dict(leaves)
    for tw in twigs:
        tot = 0
        for key, c in kids[tw]:
            del want[key]
            tot += c
        want[tw] = tot
    assert _leaves(T2) == want
    assert T2.L == T.L - sum(len(kids[t]) for t in twigs) + len(twigs)


def test_pushdown_matches_brute_force_octants():
    T, (xs, ys, zs) = _tree()
    lo, k = T.lo, T.k
    qx, qy, qz = _q(xs, lo[0], k), _q(ys, lo[1], k), _q(zs, lo[2], k)
    order = np.argsort(-T.leaf_count, kind="stable")[:5]
    edits, want = [], _leaves(T)
    for li in order:
        l, p, b, c = int(T.leaf_level[li]), int(T.leaf_prefix[li]), int(T.leaf_start[li]), int(T.leaf_count[li])
        edits.append((l, p, 2))
        del want[(l, p)]
        sh = 20 - l
        o = ((qx[b:b + c] >> sh) & 1) | (((qy[b:b + c] >> sh) & 1) << 1) | (((qz[b:b + c] >> sh) & 1) << 2)
        for oc in range(8):
            cnt = int((o == oc).sum())
            if cnt:
                want[(l + 1, (p << 3) | oc)] = cnt
    T2 = T.rebuild(xs, ys, zs, mode=2, edits=edits)
    _valid(T2)
    assert _leaves(T2) == want


def test_inverse_edits_restore_the_tree():
    T, (xs, ys, zs) = _tree()
    li = int(np.argmax(T.leaf_count))
    l, p = int(T.leaf_level[li]), int(T.leaf_prefix[li])
    T2 = T.rebuild(xs, ys, zs, mode=2, edits=[(l, p, 2)])
    assert T2.L > T.L
    T3 = T2.rebuild(xs, ys, zs, mode=2, edits=[(l, p, 1)])
    for a in ("leaf_count", "leaf_level", "leaf_prefix", "u_off", "u_idx"):
        assert np.array_equal(getattr(T3, a), getattr(T, a))


def test_collapse_root_and_absent_nodes():
    T, (xs, ys, zs) = _tree()
    R = T.rebuild(xs, ys, zs, mode=2, edits=[(0, 0, 1)])
    assert R.L == 1 and R.leaf_count[0] == T.n
    # edits naming nodes that do not exist change nothing
    ghost = [(3, (1 << 9) + 7, 1), (21, 12345, 2)]
    existing = {(int(l), int(p)) for l, p in zip(T.node_level, T.node_prefix)}
    assert not any((l, p) in existing for l, p, _ in ghost)
    G = T.rebuild(xs, ys, zs, mode=2, edits=ghost)
    assert np.array_equal(G.leaf_prefix, T.leaf_prefix) and np.array_equal(G.leaf_count, T.leaf_count)


def test_keep_after_motion_keeps_parents():
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(12000, 5)
    dom = synth.c5_domain(x, y, z)
    T = oracle.Tree(x, y, z, 24, domain=dom)
    px, py, pz, vx, vy, vz = (a[T.perm] for a in (x, y, z, vx, vy, vz))
    px, py, pz = oracle.drift(px, py, pz, vx, vy, vz, 0.05)
    T2 = T.rebuild(px, py, pz, mode=2)
    _valid(T2)
    old_int, new_int = _internal(T), _internal(T2)
    assert new_int <= old_int                                   # no new parents
    nodes2 = {(int(l), int(p)) for l, p in zip(T2.node_level, T2.node_prefix)}
    assert old_int & nodes2 <= new_int                          # surviving parents stay parents
    # the moved bodies really changed the leaves (the test is not vacuous)
    assert not np.array_equal(T2.leaf_count, T.leaf_count[:T2.L]) or T2.L != T.L


def test_enforce_mode_equals_enforce_with_edits_overriding():
    T, (xs, ys, zs) = _tree()
    E = T.enforce(xs, ys, zs, S=40)
    R = T.rebuild(xs, ys, zs, S=40, mode=1)
    assert np.array_equal(E.leaf_prefix, R.leaf_prefix) and np.array_equal(E.leaf_count, R.leaf_count)
    # a PushDown edit beats the Enforce_S rule for that node
    li = int(np.argmax(R.leaf_count))
    l, p = int(R.leaf_level[li]), int(R.leaf_prefix[li])
    R2 = T.rebuild(xs, ys, zs, S=40, mode=1, edits=[(l, p, 2)])
    assert (l, p) not in _leaves(R2) and R2.L > R.L
