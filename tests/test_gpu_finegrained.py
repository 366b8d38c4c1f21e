"""FineGrainedOptimize on the GPU (PAPER L20 SVI.B):
afmm_tree_rebuild (KEEP / ENFORCE + Collapse / PushDown edits) bit-exact with
oracle_tree_rebuild, the far-field operation counts M(Op) bit-exact with
oracle_farfield_counts, and afmm_fine_grained's contract (the prediction never
gets worse, a rejected group is undone exactly, the returned tree's predicted
time is the one reported)."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

KEYS = ("perm", "leaf_start", "leaf_count", "leaf_level", "leaf_prefix", "u_off", "u_idx")


def _afmm():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    return afmm


def _dev(*a):
    return [torch.from_numpy(np.ascontiguousarray(v)).cuda() for v in a]


def _same(G, To, tag):
    for k in KEYS:
        assert np.array_equal(G[k], getattr(To, k)), (tag, k)


def _edits(To, rng, n_collapse=9, n_push=9):
    """Collapse random twigs and push down random leaves, plus absent nodes."""
    leaf = {(int(l), int(p)) for l, p in zip(To.leaf_level, To.leaf_prefix)}
    nchild, nleafkids = {}, {}
    for l, p in zip(To.node_level, To.node_prefix):
        if l > 0:
            par = (int(l) - 1, int(p) >> 3)
            nchild[par] = nchild.get(par, 0) + 1
            if (int(l), int(p)) in leaf:
                nleafkids[par] = nleafkids.get(par, 0) + 1
    twigs = sorted(k for k, c in nchild.items() if nleafkids.get(k, 0) == c)
    big = [(int(l), int(p)) for l, p, c in zip(To.leaf_level, To.leaf_prefix, To.leaf_count) if c >= 2]
    ed = [(l, p, 1) for l, p in (twigs[i] for i in rng.choice(len(twigs), n_collapse, replace=False))]
    ed += [(l, p, 2) for l, p in (big[i] for i in rng.choice(len(big), n_push, replace=False))]
    ed += [(4, 4095, 1), (21, 7, 2)]                       # absent nodes: no effect
    rng.shuffle(ed)
    return [tuple(map(int, e)) for e in ed]


@pytest.mark.parametrize("mode", [1, 2])
def test_rebuild_with_edits_bit_exact(mode):
    afmm = _afmm()
    rng = np.random.default_rng(11 + mode)
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(80000, 5)
    dom = synth.c5_domain(x, y, z)
    S = 32
    t = afmm.GpuTree(0)
    t.build(*_dev(x, y, z), S, domain=dom)
    To = oracle.Tree(x, y, z, S, domain=dom)
    px, py, pz, qx, qy, qz = (a[To.perm] for a in (x, y, z, vx, vy, vz))
    for step in range(4):
        px, py, pz = oracle.drift(px, py, pz, qx, qy, qz, 0.3)
        ed = _edits(To, rng)
        S2 = S + 8 * (step % 2)
        t.rebuild(*_dev(px, py, pz), S2, mode=mode, edits=ed)
        To2 = To.rebuild(px, py, pz, S=S2, mode=mode, edits=ed)
        _same(t.copy_out(80000), To2, (mode, step))
        nd = t.nodes()
        o = np.lexsort((To2.node_prefix, To2.node_level))
        assert np.array_equal(nd["prefix"], To2.node_prefix[o]) and np.array_equal(nd["level"], To2.node_level[o])
        assert np.array_equal(t.farfield_counts(), To2.farfield_counts()), (mode, step)
        px, py, pz, qx, qy, qz = (a[To2.perm] for a in (px, py, pz, qx, qy, qz))
        To = To2
    t.close()


def test_nodes_export_matches_oracle():
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", 50000, 9)
    t = afmm.GpuTree(0)
    t.build(*_dev(x, y, z), 40)
    To = oracle.Tree(x, y, z, 40, ulist=False)
    nd = t.nodes()
    o = np.lexsort((To.node_prefix, To.node_level))          # level-major, ascending prefix
    assert np.array_equal(nd["level"], To.node_level[o])
    assert np.array_equal(nd["prefix"], To.node_prefix[o])
    assert np.array_equal(nd["nchild"] == 0, To.node_is_leaf[o].astype(bool))
    t.close()


@pytest.mark.parametrize("dist,n,S", [("uniform", 4096, 64), ("plummer", 200000, 128), ("colliding", 150000, 96)])
def test_farfield_counts_vs_oracle(dist, n, S):
    afmm = _afmm()
    x, y, z, m = synth.make(dist, n, 3)
    t = afmm.GpuTree(0)
    t.build(*_dev(x, y, z), S)
    To = oracle.Tree(x, y, z, S)
    assert np.array_equal(t.farfield_counts(), To.farfield_counts())
    t.close()


def _predict(counts, coef):
    return max(float(np.dot(coef[:5], counts[:5])), float(coef[5] * counts[5]))


@pytest.mark.parametrize("direction", [1, -1])
def test_fine_grained_improves_prediction(direction):
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", 200000, 4)
    X, Y, Z = _dev(x, y, z)
    t = afmm.GpuTree(0)
    t.build(X, Y, Z, 128)
    c0 = t.farfield_counts().astype(np.float64)
    # per-op costs chosen so the requested side runs ~2x longer than the other
    cpu0 = float(c0[:5].sum())
    coef = np.ones(6)
    if direction > 0:
        coef[5] = cpu0 / (2.0 * c0[5])
    else:
        coef[5] = 2.0 * cpu0 / c0[5]
    t0 = _predict(c0, coef)
    r = t.fine_grained(X, Y, Z, 128, coef, direction=0, group_frac=0.05, max_groups=32)
    assert r["direction"] == direction
    assert r["t_before"] == pytest.approx(t0, rel=1e-12)
    assert r["groups_applied"] >= 1 and r["t_after"] < r["t_before"]
    c1 = t.farfield_counts()
    assert _predict(c1, coef) == pytest.approx(r["t_after"], rel=1e-12)
    G = t.copy_out(200000)
    assert int(G["leaf_count"].sum()) == 200000
    assert G["leaf_start"][0] == 0 and (G["leaf_start"][1:] == G["leaf_start"][:-1] + G["leaf_count"][:-1]).all()
    t.close()


def test_fine_grained_rejected_group_is_undone():
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", 100000, 4)
    X, Y, Z = _dev(x, y, z)
    t = afmm.GpuTree(0)
    t.build(X, Y, Z, 64)
    before = t.copy_out(100000)
    c0 = t.farfield_counts()
    # P2P-only cost: collapsing can only raise the prediction -> first group rejected
    coef = np.array([0, 0, 0, 0, 0, 1.0])
    r = t.fine_grained(X, Y, Z, 64, coef, direction=1, group_frac=0.1, max_groups=4)
    assert r["groups_tried"] == 1 and r["groups_applied"] == 0 and r["t_after"] == r["t_before"]
    after = t.copy_out(100000)
    for k in KEYS:
        assert np.array_equal(after[k], before[k]), k
    assert np.array_equal(t.farfield_counts(), c0)
    t.close()
