"""Pins for the fp64 oracle (CPU only).  Each pin checks the oracle against
something other than itself: brute force written without tree code, closed
forms, a lattice with a closed-form U-list, invariants of the definitions in
PAPER.md L10 SI.B (tree), L12 SI.C (near field / P2P), L16 SIII.C
(Interactions(t), GPU split).  See DESIGN.md "Oracle pins"."""
import numpy as np
import pytest

import oracle
import synth

G = 1.0


def _bruteforce_allpairs(x, y, z, m, eps2, G=1.0):
    """Textbook O(N^2) direct sum, no tree code, j != i (numpy, fp64)."""
    p = np.stack([x, y, z], 1).astype(np.float64)
    mm = m.astype(np.float64)
    d = p[None, :, :] - p[:, None, :]                  # d[i, j] = x_j - x_i
    r2 = (d ** 2).sum(-1) + eps2
    np.fill_diagonal(r2, 1.0)
    inv = 1.0 / np.sqrt(r2)
    np.fill_diagonal(inv, 0.0)
    phi = -(G * mm[None, :] * inv).sum(1)
    a = (G * mm[None, :, None] * (inv ** 3)[:, :, None] * d).sum(1)
    return phi, a[:, 0], a[:, 1], a[:, 2]


def _rel(a, b):
    return np.abs(a - b).max() / max(np.abs(b).max(), 1e-300)


# ----------------------------------------------------------------- special cases

def test_single_leaf_equals_allpairs():
    """N <= S: the root is the only leaf, U(root) = {root}: P2P = all pairs."""
    x, y, z, m = synth.plummer(300, seed=11)
    T = oracle.Tree(x, y, z, S=300)
    assert T.L == 1 and list(T.u_idx) == [0] and T.leaf_level[0] == 0
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    got = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, G, 1e-4)
    ref = _bruteforce_allpairs(xs, ys, zs, ms, 1e-4)
    for g, r in zip(got, ref):
        assert _rel(g, r) < 1e-13


def test_depth1_octants_mutually_adjacent():
    """S < N with every octant <= S: 8 level-1 leaves sharing the cube centre,
    each adjacent to all others, so P2P is all-pairs again."""
    rng = np.random.default_rng(5)
    pts = []
    for o in range(8):
        off = np.array([(o >> 0) & 1, (o >> 1) & 1, (o >> 2) & 1], float) * 0.5
        pts.append(off + 0.05 + 0.4 * rng.random((20, 3)))
    pts = np.concatenate(pts)
    pts[0] = [0.0, 0.0, 0.0]
    pts[140] = [0.99, 0.99, 0.99]        # (an octant-7 body) fixes the domain to the unit cube
    x, y, z = (pts[:, c].astype(np.float32) for c in range(3))
    m = np.full(160, 1 / 160, np.float32)
    T = oracle.Tree(x, y, z, S=20)
    assert T.L == 8 and (T.leaf_level == 1).all() and (T.leaf_count == 20).all()
    assert T.u_idx.size == 64
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    got = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, G, 1e-6)
    ref = _bruteforce_allpairs(xs, ys, zs, ms, 1e-6)
    for g, r in zip(got, ref):
        assert _rel(g, r) < 1e-13


def test_two_body_closed_form():
    """a_1 = G m_2 d / (d^2+eps^2)^{3/2},  phi_1 = -G m_2 / sqrt(d^2+eps^2)."""
    x = np.array([0.25, 0.75], np.float32)
    y = np.array([0.5, 0.125], np.float32)
    z = np.array([0.0, 0.5], np.float32)
    m = np.array([0.5, 0.25], np.float32)
    T = oracle.Tree(x, y, z, S=4)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    for eps2 in (0.0, 1e-2):
        phi, ax, ay, az, A = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off,
                                        T.u_idx, 2.0, eps2, with_scale=True)
        for i in range(2):
            j = 1 - i
            d = np.array([xs[j] - xs[i], ys[j] - ys[i], zs[j] - zs[i]], float)
            r2 = float(d @ d) + eps2
            assert phi[i] == pytest.approx(-2.0 * ms[j] / np.sqrt(r2), rel=1e-15)
            exp_a = 2.0 * ms[j] * d / r2 ** 1.5
            assert np.allclose([ax[i], ay[i], az[i]], exp_a, rtol=1e-15, atol=0)
            assert A[i] == pytest.approx(2.0 * ms[j] * np.sqrt(d @ d) / r2 ** 1.5, rel=1e-15)


def test_single_body_is_zero():
    x, y, z, m = (np.array([v], np.float32) for v in (0.3, 0.4, 0.5, 1.0))
    T = oracle.Tree(x, y, z, S=1)
    phi, ax, ay, az = oracle.p2p(x, y, z, m, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, G, 0.0)
    assert phi[0] == 0.0 and ax[0] == 0.0 and ay[0] == 0.0 and az[0] == 0.0


def test_coincident_bodies_eps0_is_nonfinite():
    """Reading R21: eps2 = 0 with two distinct coincident bodies gives inf/NaN."""
    x = np.array([0.5, 0.5, 0.1], np.float32)
    y = np.array([0.5, 0.5, 0.2], np.float32)
    z = np.array([0.5, 0.5, 0.3], np.float32)
    m = np.ones(3, np.float32)
    T = oracle.Tree(x, y, z, S=8)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    phi, *_ = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, G, 0.0)
    assert not np.isfinite(phi).all()


# ----------------------------------------------------------------- tree invariants

def _deinterleave(prefix, level):
    q = np.zeros((prefix.shape[0], 3), np.int64)
    for b in range(int(level.max()) if level.size else 0):
        use = level > b
        for a in range(3):
            bit = ((prefix >> np.uint64(3 * b + a)) & np.uint64(1)).astype(np.int64)
            q[:, a] |= np.where(use, bit << b, 0)
    return q


def _leaf_boxes(T):
    q = _deinterleave(T.leaf_prefix, T.leaf_level)
    w = (np.int64(1) << (21 - T.leaf_level.astype(np.int64)))
    return q * w[:, None], w


@pytest.mark.parametrize("dist,n,S,seed", [("uniform", 4096, 64, 1), ("plummer", 20000, 32, 7),
                                           ("colliding", 20000, 50, 9), ("plummer", 3000, 1, 3)])
def test_tree_invariants(dist, n, S, seed):
    x, y, z, m = synth.make(dist, n, seed)
    T = oracle.Tree(x, y, z, S, ulist=False)
    # domain: side = 2^k is the smallest power of two strictly above the extent
    P = np.stack([x, y, z], 1).astype(np.float64)
    ext = (P.max(0) - P.min(0)).max()
    assert np.array_equal(T.lo, P.min(0))
    assert 2.0 ** T.k > ext and (ext == 0 or 2.0 ** (T.k - 1) <= ext)
    # perm is a permutation; leaves tile [0, N) in order; no empty leaf
    assert np.array_equal(np.sort(T.perm), np.arange(n))
    assert T.leaf_start[0] == 0 and (T.leaf_count > 0).all()
    assert np.array_equal(T.leaf_start[1:], T.leaf_start[:-1] + T.leaf_count[:-1])
    assert T.leaf_start[-1] + T.leaf_count[-1] == n
    # capacity: count <= S unless at the maximum level 21
    assert ((T.leaf_count <= S) | (T.leaf_level == 21)).all()
    # maximality: every internal node holds more than S bodies ("more than", L10 SI.B)
    internal = T.node_is_leaf == 0
    assert ((T.node_e - T.node_b)[internal] > S).all()
    # every body lies inside its leaf's box (closed-open, in real coordinates)
    A, w = _leaf_boxes(T)
    h = 2.0 ** (T.k - 21)
    owner = np.repeat(np.arange(T.L), T.leaf_count)
    Ps = P[T.perm]
    for a in range(3):
        lo_edge = T.lo[a] + A[owner, a] * h
        hi_edge = T.lo[a] + (A[owner, a] + w[owner]) * h
        inside = (Ps[:, a] >= lo_edge) & ((Ps[:, a] < hi_edge) | (A[owner, a] + w[owner] == 2 ** 21))
        assert inside.all()
    # leaf index order = Morton order of the leaf boxes (disjoint, ascending)
    lvl = T.leaf_level.astype(np.uint64)
    first = T.leaf_prefix << (np.uint64(3) * (np.uint64(21) - lvl))
    last = first + (np.uint64(1) << (np.uint64(3) * (np.uint64(21) - lvl))) - np.uint64(1)
    assert (first[1:] > last[:-1]).all()
    # stable order: equal-position bodies keep input order
    key = np.lexsort((np.arange(n), Ps[:, 2], Ps[:, 1], Ps[:, 0]))   # tree position breaks ties
    dup = np.all(Ps[key[1:]] == Ps[key[:-1]], axis=1)
    assert (T.perm[key[1:]][dup] > T.perm[key[:-1]][dup]).all()


def test_tree_stable_for_duplicate_positions():
    """Reading R10: bodies with equal Morton keys keep their input order."""
    x, y, z, m = synth.make("uniform", 500, 3)
    idx = np.arange(500) % 50                  # every position appears 10 times
    x, y, z = x[idx], y[idx], z[idx]
    T = oracle.Tree(x, y, z, 4, ulist=False)
    Ps = np.stack([x, y, z], 1)[T.perm]
    for p in range(1, 500):
        if (Ps[p] == Ps[p - 1]).all():
            assert T.perm[p] > T.perm[p - 1]
    assert (T.leaf_level[T.leaf_count > 4] == 21).all()


# ----------------------------------------------------------------- U-list

def _adjacent_boxes(A, w):
    """Independent closed-box adjacency matrix over all leaves (O(L^2))."""
    ok = np.ones((A.shape[0], A.shape[0]), bool)
    for a in range(3):
        ok &= (A[:, None, a] <= A[None, :, a] + w[None, :]) & (A[None, :, a] <= A[:, None, a] + w[:, None])
    return ok


@pytest.mark.parametrize("dist,n,S,seed", [("uniform", 4096, 64, 1), ("plummer", 6000, 16, 2),
                                           ("colliding", 6000, 24, 4)])
def test_ulist_complete_symmetric_sorted(dist, n, S, seed):
    x, y, z, m = synth.make(dist, n, seed)
    T = oracle.Tree(x, y, z, S)
    A, w = _leaf_boxes(T)
    adj = _adjacent_boxes(A, w)
    dense = np.zeros((T.L, T.L), bool)
    rows = np.repeat(np.arange(T.L), np.diff(T.u_off))
    dense[rows, T.u_idx] = True
    assert np.array_equal(dense, adj)                   # complete and exact
    assert np.array_equal(dense, dense.T)               # symmetric
    assert dense.diagonal().all()                       # contains self (reading R5)
    for t in range(T.L):
        r = T.u_idx[T.u_off[t]:T.u_off[t + 1]]
        assert (np.diff(r) > 0).all()                   # strictly ascending


@pytest.mark.parametrize("M", [2, 4, 8, 16])
def test_ulist_lattice_closed_form(M):
    """One body per cell centre of an M^3 grid, S = 1: every leaf is at level
    log2 M; nnz = (3M-2)^3; row size = prod over axes of |{i-1,i,i+1} cap [0,M)|."""
    x, y, z, m = synth.lattice(M)
    T = oracle.Tree(x, y, z, S=1)
    lev = int(np.log2(M))
    assert T.L == M ** 3 and (T.leaf_level == lev).all() and (T.leaf_count == 1).all()
    assert T.u_idx.size == (3 * M - 2) ** 3
    A, w = _leaf_boxes(T)
    cell = A // w[:, None]
    per_axis = np.where((cell == 0) | (cell == M - 1), 2, 3)
    if M == 1:
        per_axis[:] = 1
    assert np.array_equal(np.diff(T.u_off), per_axis.prod(1))


# ----------------------------------------------------------------- P2P vs brute force

def test_c1_bruteforce_with_independent_adjacency():
    """C1 (4096 uniform, S=64): every ordered pair (i, j), i != j, whose leaf
    boxes touch contributes; checked against the oracle to 1e-13 and the pair
    count against sum_t Interactions(t) exactly."""
    x, y, z, m = synth.make("C1")
    eps2 = 1e-6
    T = oracle.Tree(x, y, z, 64)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    got = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, G, eps2)
    A, w = _leaf_boxes(T)
    owner = np.repeat(np.arange(T.L), T.leaf_count)
    Ab, wb = A[owner], w[owner]
    P = np.stack([xs, ys, zs], 1).astype(np.float64)
    n = P.shape[0]
    phi = np.zeros(n)
    acc = np.zeros((n, 3))
    pairs = 0
    for i0 in range(0, n, 512):
        sl = slice(i0, min(n, i0 + 512))
        adj = np.ones((sl.stop - i0, n), bool)
        for a in range(3):
            adj &= (Ab[sl, None, a] <= Ab[None, :, a] + wb[None, :]) & (Ab[None, :, a] <= Ab[sl, None, a] + wb[sl, None])
        pairs += int(adj.sum())
        adj[np.arange(sl.stop - i0), np.arange(i0, sl.stop)] = False
        d = P[None, :, :] - P[sl, None, :]
        r2 = (d ** 2).sum(-1) + eps2
        inv = np.where(adj, 1.0 / np.sqrt(r2), 0.0)
        phi[sl] = -(ms.astype(np.float64)[None, :] * inv).sum(1)
        acc[sl] = (ms.astype(np.float64)[None, :, None] * (inv ** 3)[:, :, None] * d).sum(1)
    assert _rel(got[0], phi) < 1e-13
    for c in range(3):
        assert _rel(got[1 + c], acc[:, c]) < 1e-12
    I = oracle.interactions(T.leaf_count, T.u_off, T.u_idx)
    assert int(I.sum()) == pairs


def test_newton_third_law_and_energy_symmetry():
    """U symmetric => sum_i m_i a_i = 0 and sum_i m_i phi_i = 2 sum_{pairs} -G m_i m_j / r."""
    x, y, z, m = synth.plummer(8000, seed=21)
    m = (m * (1.0 + np.arange(8000) % 7)).astype(np.float32)      # unequal masses
    T = oracle.Tree(x, y, z, 40)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    phi, ax, ay, az, A = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx,
                                    G, 1e-6, with_scale=True)
    mm = ms.astype(np.float64)
    scale = (mm * A).sum()
    for a in (ax, ay, az):
        assert abs((mm * a).sum()) <= 1e-12 * scale
    # pair energy via the U-list CSR (each unordered adjacent pair once, i<j)
    P = np.stack([xs, ys, zs], 1).astype(np.float64)
    E = 0.0
    for t in range(T.L):
        it = np.arange(T.leaf_start[t], T.leaf_start[t] + T.leaf_count[t])
        for s in T.u_idx[T.u_off[t]:T.u_off[t + 1]]:
            js = np.arange(T.leaf_start[s], T.leaf_start[s] + T.leaf_count[s])
            d = P[js][None, :, :] - P[it][:, None, :]
            r = np.sqrt((d ** 2).sum(-1) + 1e-6)
            keep = js[None, :] > it[:, None]
            E += (np.where(keep, -mm[it][:, None] * mm[js][None, :] / r, 0.0)).sum()
    assert (mm * phi).sum() == pytest.approx(2 * E, rel=1e-12)


def test_mass_scaling_bit_exact():
    x, y, z, m = synth.make("C1")
    T = oracle.Tree(x, y, z, 64)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    a = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, G, 1e-6)
    b = oracle.p2p(xs, ys, zs, (ms * np.float32(8)).astype(np.float32), T.leaf_start,
                   T.leaf_count, T.u_off, T.u_idx, G, 1e-6)
    for u, v in zip(a, b):
        assert np.array_equal(v, u * 8)


def test_target_subset_matches_full():
    x, y, z, m = synth.make("C1")
    T = oracle.Tree(x, y, z, 64)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    full = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, G, 1e-6)
    tg = np.array([0, 7, T.L - 1], np.int32)
    sub = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, G, 1e-6,
                     targets=tg)
    for t in tg:
        sl = slice(T.leaf_start[t], T.leaf_start[t] + T.leaf_count[t])
        for u, v in zip(full, sub):
            assert np.array_equal(u[sl], v[sl])


# ----------------------------------------------------------------- partition

@pytest.mark.parametrize("Gp", [1, 2, 3, 4, 8])
def test_partition_literal_invariants(Gp):
    """L16 SIII.C: GPUs 0..G-2 each receive the shortest prefix of the remaining
    leaves whose count meets or exceeds total/G; the last GPU gets the rest."""
    x, y, z, m = synth.make("plummer", 20000, 3)
    T = oracle.Tree(x, y, z, 32)
    I = oracle.interactions(T.leaf_count, T.u_off, T.u_idx)
    owner, split = oracle.partition_literal(I, Gp)
    total = int(I.sum())
    assert split[0] == 0 and split[-1] == T.L and (np.diff(split) >= 0).all()
    assert (np.diff(owner) >= 0).all() and (np.diff(owner) <= 1).all()
    for r in range(Gp):
        assert (owner[split[r]:split[r + 1]] == r).all()
    for r in range(Gp - 1):
        c = int(I[split[r]:split[r + 1]].sum())
        assert c * Gp >= total                                    # meets or exceeds
        if split[r + 1] > split[r]:
            assert (c - int(I[split[r + 1] - 1])) * Gp < total    # and is the first to do so


def test_partition_more_gpus_than_leaves():
    I = np.array([5, 1, 1], np.int64)
    owner, split = oracle.partition_literal(I, 8)
    assert list(split) == [0, 1, 2, 3, 3, 3, 3, 3, 3]


# ----------------------------------------------------------------- generators

def test_plummer_radial_cdf():
    """Generator sanity: the truncated Plummer radial CDF r^3/(1+r^2)^{3/2}."""
    x, y, z, m = synth.plummer(200000, seed=1)
    r = np.sqrt(x.astype(float) ** 2 + y.astype(float) ** 2 + z.astype(float) ** 2)
    assert r.max() <= 10.0 + 1e-5
    Mr = lambda q: q ** 3 / (1 + q ** 2) ** 1.5
    for q in (0.5, 1.0, 2.0, 5.0):
        assert np.mean(r <= q) == pytest.approx(Mr(q) / Mr(10.0), abs=5e-3)
    assert m.sum() == pytest.approx(1.0, rel=1e-6)


def test_generators_deterministic():
    a = synth.make("C1")
    b = synth.make("C1")
    for u, v in zip(a, b):
        assert np.array_equal(u, v)
    c = synth.make("uniform", 4096, 2)
    assert not np.array_equal(a[0], c[0])
