"""The split rule the GPU's direct tree construction relies on (csrc/tree_build.cu
section 4d, DESIGN.md section 6 "Leaves and nodes"), restated on the sorted keys
and checked here on the CPU against the oracle's recursive split (reading R7) and
its Collapse / PushDown walk (Enforce_S, reading R22):

  the node at level l holding sorted body i has more than S bodies iff some window
  of S + 1 consecutive sorted keys containing i shares its first l octal digits,

so with w_j = lcp(key_j, key_{j+S}) and M_i = max of w_j over the windows that
contain i, body i's leaf is at level min(M_i + 1, 21) (the root if no window),
deepened by Enforce_S while the node holds exactly S bodies (the same maxima over
windows of S) and was a parent in the previous tree; a leaf starts at i iff
lcp(key_{i-1}, key_i) < that level.  numpy only (no GPU); the keys follow R10."""
import numpy as np
import pytest
from numpy.lib.stride_tricks import sliding_window_view

import oracle
import synth

K = 21


def morton_keys(x, y, z, lo, k):
    """R10: q = clamp(floor((x - lo) 2^(21-k)), 0, 2^21 - 1) in fp64; bit b of q_x/q_y/q_z -> key bits 3b/3b+1/3b+2."""
    scale = np.ldexp(1.0, K - k)
    q = [np.clip(np.floor((v.astype(np.float64) - lo[a]) * scale), 0, 2 ** K - 1).astype(np.uint64)
         for a, v in enumerate((x, y, z))]
    key = np.zeros(x.shape[0], np.uint64)
    for b in range(K):
        for a in range(3):
            key |= ((q[a] >> np.uint64(b)) & np.uint64(1)) << np.uint64(3 * b + a)
    return key


def lcp_digits(a, b):
    """Leading octal digits (of 21) two 63-bit keys share."""
    x = a ^ b
    bitlen = np.zeros(x.shape, np.int64)
    for s in range(64):
        bitlen += (x >> np.uint64(s)) != 0
    return np.where(x == 0, K, (63 - bitlen) // 3)


def window_max(w, S, n, width):
    """max of w_j over the windows [j, j + width] (width = S: windows of S + 1 keys) containing each i; -1 if none."""
    pad = np.full(width, -1, np.int64)
    wp = np.concatenate([pad, w, np.full(n - w.shape[0], -1, np.int64)])
    return sliding_window_view(wp, width + 1).max(axis=1)[:n]


def leaves_by_rule(key, S, prev_internal=None):
    n = key.shape[0]
    w = lcp_digits(key[:max(n - S, 0)], key[S:]) if n > S else np.zeros(0, np.int64)
    m1 = window_max(w, S, n, S)                               # windows of S + 1 keys
    lvl = np.where(m1 < 0, 0, np.minimum(m1 + 1, K))
    if prev_internal is not None:
        v = lcp_digits(key[:n - S + 1], key[S - 1:]) if n >= S else np.zeros(0, np.int64)
        m2 = window_max(v, S, n, S - 1)                       # windows of S keys
        for i in range(n):
            lv = int(lvl[i])
            while lv < K and lv <= m2[i] and (lv, int(key[i] >> np.uint64(3 * (K - lv)))) in prev_internal:
                lv += 1
            lvl[i] = lv
    start = np.ones(n, bool)
    start[1:] = lcp_digits(key[:-1], key[1:]) < lvl[1:]
    ls = np.flatnonzero(start)
    ll = lvl[ls]
    lp = np.array([int(key[i]) >> (3 * (K - int(l))) for i, l in zip(ls, ll)], np.uint64)
    return ls.astype(np.int32), ll.astype(np.int32), lp


def sorted_keys(x, y, z, T):
    key = morton_keys(x, y, z, T.lo, T.k)
    order = np.lexsort((np.arange(key.shape[0]), key))       # stable by (key, index)
    assert np.array_equal(order, T.perm)
    return key[order]


@pytest.mark.parametrize("dist,n,S,seed", [("plummer", 20000, 32, 1), ("uniform", 5000, 64, 2),
                                           ("colliding", 20000, 17, 3), ("plummer", 3000, 1, 4),
                                           ("uniform", 50, 64, 5), ("uniform", 64, 64, 6)])
def test_fresh_split_rule_matches_oracle(dist, n, S, seed):
    x, y, z, m = synth.make(dist, n, seed)
    T = oracle.Tree(x, y, z, S, ulist=False)
    ls, ll, lp = leaves_by_rule(sorted_keys(x, y, z, T), S)
    assert np.array_equal(ls, T.leaf_start)
    assert np.array_equal(ll, T.leaf_level)
    assert np.array_equal(lp, T.leaf_prefix)


def test_fresh_rule_duplicate_keys_level21():
    """Identical keys: leaves stop at level 21 above S (R8)."""
    x, y, z, m = synth.make("uniform", 600, 3)
    idx = np.arange(600) % 40
    x, y, z = x[idx], y[idx], z[idx]
    T = oracle.Tree(x, y, z, 4, ulist=False)
    ls, ll, lp = leaves_by_rule(sorted_keys(x, y, z, T), 4)
    assert np.array_equal(ls, T.leaf_start) and np.array_equal(ll, T.leaf_level)
    assert (ll == K).any()


@pytest.mark.parametrize("S", [8, 16, 33])
def test_enforce_rule_matches_oracle_walk(S):
    """Enforce_S along a short trajectory: the rule with the 'exactly S and was a
    parent' extension equals the oracle's Collapse / PushDown walk, and the walk
    differs from a fresh build at some step (the extension is exercised)."""
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(6000, 5)
    dom = synth.c5_domain(x, y, z)
    To = oracle.Tree(x, y, z, S, domain=dom, ulist=False)
    px, py, pz, qx, qy, qz = (a[To.perm] for a in (x, y, z, vx, vy, vz))
    differs = 0
    for step in range(6):
        px, py, pz = oracle.drift(px, py, pz, qx, qy, qz, 0.5)
        To2 = To.enforce(px, py, pz, S, ulist=False)
        prev_internal = {(int(l), int(p)) for l, p, lf in zip(To.node_level, To.node_prefix, To.node_is_leaf)
                         if not lf}
        key = sorted_keys(px, py, pz, To2)
        ls, ll, lp = leaves_by_rule(key, S, prev_internal)
        assert np.array_equal(ls, To2.leaf_start), step
        assert np.array_equal(ll, To2.leaf_level), step
        assert np.array_equal(lp, To2.leaf_prefix), step
        fresh = leaves_by_rule(key, S)
        differs += int(fresh[0].shape != ls.shape or not np.array_equal(fresh[0], ls))
        px, py, pz, qx, qy, qz = (a[To2.perm] for a in (px, py, pz, qx, qy, qz))
        To = To2
    assert differs > 0
