"""GPU octree + U-list builder (include/afmm_tree.h) vs the oracle: bit-exact
integer indexing (perm, leaves, levels, prefixes, CSR U-lists), plus the
full-size configs end to end (GPU tree -> GPU P2P) checked on sampled leaves."""
import numpy as np
import pytest

import oracle
import synth
from tests import _tol

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _afmm():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    return afmm


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.float32)).cuda()


def gpu_tree(x, y, z, S, domain=None):
    afmm = _afmm()
    t = afmm.GpuTree(0)
    t.build(_dev(x), _dev(y), _dev(z), S, domain=domain)
    out = t.copy_out(x.shape[0])
    t.close()
    return out


def assert_same_tree(G, T):
    assert G["n_leaves"] == T.L
    assert G["k"] == T.k and np.array_equal(G["lo"], T.lo)
    assert np.array_equal(G["perm"], T.perm)
    assert np.array_equal(G["leaf_start"], T.leaf_start)
    assert np.array_equal(G["leaf_count"], T.leaf_count)
    assert np.array_equal(G["leaf_level"], T.leaf_level)
    assert np.array_equal(G["leaf_prefix"], T.leaf_prefix)
    assert np.array_equal(G["u_off"], T.u_off)
    assert np.array_equal(G["u_idx"], T.u_idx)


@pytest.mark.parametrize("dist,n,S,seed", [("uniform", 4096, 64, 1), ("plummer", 100000, 32, 2),
                                           ("colliding", 100000, 100, 3), ("plummer", 50000, 1, 4),
                                           ("uniform", 1, 4, 5), ("uniform", 300, 500, 6),
                                           ("plummer", 1 << 20, 128, 2)])
def test_tree_bit_exact(dist, n, S, seed):
    x, y, z, m = synth.make(dist, n, seed)
    assert_same_tree(gpu_tree(x, y, z, S), oracle.Tree(x, y, z, S))


def test_tree_lattice_and_duplicates_bit_exact():
    x, y, z, m = synth.lattice(16)
    assert_same_tree(gpu_tree(x, y, z, 1), oracle.Tree(x, y, z, 1))
    x, y, z, m = synth.make("uniform", 600, 3)
    idx = np.arange(600) % 40
    x, y, z = x[idx], y[idx], z[idx]
    assert_same_tree(gpu_tree(x, y, z, 4), oracle.Tree(x, y, z, 4))


def test_tree_fixed_domain_bit_exact():
    x, y, z, m = synth.make("colliding", 50000, 7)
    dom = (np.array([-40.0, -40.0, -40.0]), 7)          # side 128, some bodies clamp nowhere
    assert_same_tree(gpu_tree(x, y, z, 64, domain=dom), oracle.Tree(x, y, z, 64, domain=dom))
    dom = (np.array([-2.0, -2.0, -2.0]), 2)             # bodies outside are clamped to the edge cells
    assert_same_tree(gpu_tree(x, y, z, 64, domain=dom), oracle.Tree(x, y, z, 64, domain=dom))


def test_gather_scatter_roundtrip():
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", 10000, 1)
    t = afmm.GpuTree(0)
    X = _dev(x)
    t.build(X, _dev(y), _dev(z), 16)
    perm = t.copy_out(10000)["perm"]
    out = torch.empty_like(X)
    t.gather(X, out)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), x[perm])
    back = torch.empty_like(X)
    t.scatter(out, back)
    torch.cuda.synchronize()
    assert np.array_equal(back.cpu().numpy(), x)
    rows = torch.stack([_dev(v) for v in (x, y, z, m)])          # afmm_tree_gather_rows
    rows_out = torch.empty_like(rows)
    t.gather_rows(rows, rows_out)
    torch.cuda.synchronize()
    assert np.array_equal(rows_out.cpu().numpy(), np.stack([x, y, z, m])[:, perm])
    t.close()


def _end_to_end(cfg, n_sample_leaves, seed=0):
    """GPU tree + GPU P2P (the bench's launch configuration) at full size;
    tree checked bit-exact, P2P checked on a seeded sample of target leaves."""
    afmm = _afmm()
    c = synth.CONFIGS[cfg]
    x, y, z, m = synth.make(cfg)
    G = gpu_tree(x, y, z, c["S"])
    T = oracle.Tree(x, y, z, c["S"])
    assert_same_tree(G, T)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    h = afmm.P2P(eps2=c["eps2"])
    h.set_bodies(*[_dev(v) for v in (xs, ys, zs, ms)])
    h.set_tree(G["leaf_start"], G["leaf_count"], G["u_off"], G["u_idx"])
    out = [torch.empty(xs.shape[0], device="cuda") for _ in range(4)]
    st = h.eval(*out, stats=True)
    ax, ay, az, phi = (o.cpu().numpy() for o in out)
    got = [phi, ax, ay, az]                           # the oracle's order
    h.close()
    rng = np.random.default_rng(seed)
    tg = np.sort(rng.choice(T.L, size=min(n_sample_leaves, T.L), replace=False)).astype(np.int32)
    tg = np.unique(np.concatenate([tg, [0, T.L - 1, int(np.argmax(T.leaf_count))]])).astype(np.int32)
    ref = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, c["eps2"],
                     targets=tg, with_scale=True)
    sel = np.zeros(xs.shape[0], bool)
    for t in tg:
        sel[T.leaf_start[t]:T.leaf_start[t] + T.leaf_count[t]] = True
    _tol.check([g[sel] for g in got], [r[sel] for r in ref[:4]], ref[4][sel])
    assert np.isfinite(np.stack(got)).all()
    return st


def test_c4_end_to_end_sampled():
    """16M Plummer, S=256 (BASELINE configs[3]) on one GPU: >= 4096 sampled leaves."""
    st = _end_to_end("C4", 4096, seed=4)
    assert st["interactions_total"] > 3e10


def test_c3_end_to_end_sampled():
    _end_to_end("C3", 4096, seed=3)


def test_ulist_dfs_fallback_matches_warp_descent(monkeypatch):
    """The U-list fallback (per-thread DFS count + fill, taken when a row or frontier
    overflows the warp descent's buffers) gives the same CSR as the warp descent
    (forced with AFMM_ULIST_DFS=1), and both equal the oracle's."""
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    x, y, z, m = synth.make("plummer", 70000, 31)
    To = oracle.Tree(x, y, z, 24)
    X, Y, Z = (torch.from_numpy(v).cuda() for v in (x, y, z))
    outs = []
    for flag in ("0", "1"):
        monkeypatch.setenv("AFMM_ULIST_DFS", flag)
        t = afmm.GpuTree(0)
        t.build(X, Y, Z, 24)
        outs.append(t.copy_out(70000))
        t.close()
    for k in ("u_off", "u_idx", "leaf_start", "leaf_count"):
        assert np.array_equal(outs[0][k], outs[1][k]), k
        assert np.array_equal(outs[1][k], getattr(To, k)), k


def test_rebuild_bucket_sort_bit_exact(monkeypatch):
    """Rebuilds in the previous build's domain sort the keys by the previous leaves'
    cells (bucket_sort_kernel) instead of the full radix sort: small motions (most
    bodies stay in their cell), a large jump, and a collapse into one cell (buckets
    over the warp sort's capacity -> the full-sort fallback) all give the oracle's
    tree, as does the forced full sort (AFMM_TREE_FULL_SORT=1)."""
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    rng = np.random.default_rng(41)
    n, S = 60000, 48
    x, y, z, m = synth.make("plummer", n, 41)
    dom = (np.array([-16.0, -16.0, -16.0]), 5)
    seq = [(x, y, z)]
    for scale in (1e-3, 1e-2, 0.5):                    # drift, larger drift, a big jump
        x = (x + scale * rng.standard_normal(n)).astype(np.float32)
        y = (y + scale * rng.standard_normal(n)).astype(np.float32)
        z = (z + scale * rng.standard_normal(n)).astype(np.float32)
        seq.append((x, y, z))
    c = np.float32(0.3)                                # everything collapses into one leaf's cell
    seq.append(tuple((c + np.float32(1e-4) * rng.standard_normal(n)).astype(np.float32) for _ in range(3)))
    seq.append(seq[1])                                  # and back
    for flag in ("0", "1"):
        monkeypatch.setenv("AFMM_TREE_FULL_SORT", flag)
        t = afmm.GpuTree(0)
        for (px, py, pz) in seq:
            t.build(_dev(px), _dev(py), _dev(pz), S, domain=dom)
            assert_same_tree(t.copy_out(n), oracle.Tree(px, py, pz, S, domain=dom))
        t.close()


def _tree_and_nodes(t, n):
    G = t.copy_out(n)
    G.update({"node_" + k: v for k, v in t.nodes().items()})
    G.update({"info_" + k: v for k, v in t.info().items() if not isinstance(v, np.ndarray)})
    return G


def test_direct_construction_matches_level_loop(monkeypatch):
    """The direct construction (leaf levels from sliding windows over the sorted
    keys, nodes as the leaves' ancestors; tree_build.cu section 4d) and the
    level-synchronous split loop (AFMM_TREE_LEVELS=1) give identical trees AND
    identical node arrays (the next Enforce_S reads them), also when every device
    capacity starts tiny (AFMM_TREE_SMALL_CAPS=1: overflow, grow, rerun): fresh builds incl. S = 1,
    n <= S, duplicate keys (level-21 leaves above S), and Enforce_S chains where
    nodes hold exactly S bodies (the 'was a parent' rule), incl. at the root."""
    afmm = _afmm()
    cases = []
    x, y, z, m = synth.make("plummer", 40000, 7)
    cases.append(("plummer", (x, y, z), [("build", 16), ("enforce", 16), ("enforce", 24), ("enforce", 8)]))
    x, y, z, m = synth.make("uniform", 600, 3)
    idx = np.arange(600) % 40
    cases.append(("dups", (x[idx], y[idx], z[idx]), [("build", 4), ("enforce", 15), ("enforce", 16), ("build", 1)]))
    x, y, z, m = synth.lattice(8)
    cases.append(("lattice", (x, y, z), [("build", 1), ("enforce", 2), ("enforce", 8), ("enforce", 1)]))
    x, y, z, m = synth.make("uniform", 64, 9)
    cases.append(("root==S", (x, y, z), [("build", 32), ("enforce", 64), ("enforce", 64), ("build", 64),
                                         ("enforce", 100)]))
    x, y, z, m = synth.make("uniform", 1, 5)
    cases.append(("n=1", (x, y, z), [("build", 1), ("enforce", 1)]))
    rng = np.random.default_rng(3)
    for name, (x, y, z), ops in cases:
        n = x.shape[0]
        res = {}
        for flag, small in (("0", "0"), ("1", "0"), ("0", "1")):   # direct, level loop, direct from tiny capacities
            monkeypatch.setenv("AFMM_TREE_LEVELS", flag)
            monkeypatch.setenv("AFMM_TREE_SMALL_CAPS", small)
            t = afmm.GpuTree(0)
            px, py, pz = x, y, z
            out = []
            for step, (op, S) in enumerate(ops):
                if step > 0 and op == "enforce":        # small deterministic motion between Enforce_S calls
                    d = np.random.default_rng(step).standard_normal((3, n)).astype(np.float32) * np.float32(1e-3)
                    px, py, pz = px + d[0], py + d[1], pz + d[2]
                fn = t.build if op == "build" else t.enforce
                fn(_dev(px), _dev(py), _dev(pz), S)
                out.append(_tree_and_nodes(t, n))
            t.close()
            res[flag + small] = out
        for other in ("10", "01"):
            for step, (a, b) in enumerate(zip(res["00"], res[other])):
                assert a.keys() == b.keys()
                for k in a:
                    assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), (name, other, step, k)
    del rng


def test_enforce_graph_replay_matches_direct_launches(monkeypatch):
    """Enforce_S along a trajectory with the positions in two alternating device
    buffers (as the C5 loop holds them): the direct build captured into CUDA graphs
    and replayed (AFMM_TREE_GRAPH default) gives the same trees and node arrays as
    launching the same kernels directly (AFMM_TREE_GRAPH=0), and replays happen; the
    trees also equal the oracle's Collapse / PushDown chain."""
    afmm = _afmm()
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(50000, 6)
    dom = synth.c5_domain(x, y, z)
    S = 24
    n = x.shape[0]
    res = {}
    for flag in ("1", "0"):
        monkeypatch.setenv("AFMM_TREE_GRAPH", flag)
        t = afmm.GpuTree(0)
        bufs = [torch.empty((3, n), device="cuda") for _ in range(2)]
        t.build(_dev(x), _dev(y), _dev(z), S, domain=dom)
        To = oracle.Tree(x, y, z, S, domain=dom, ulist=False)
        px, py, pz, qx, qy, qz = (a[To.perm] for a in (x, y, z, vx, vy, vz))
        out = []
        for step in range(7):
            px, py, pz = oracle.drift(px, py, pz, qx, qy, qz, 0.3)
            b = bufs[step % 2]
            b.copy_(torch.from_numpy(np.stack([px, py, pz])))
            t.enforce(b[0], b[1], b[2], S)
            G = _tree_and_nodes(t, n)
            To2 = To.enforce(px, py, pz, S)
            for k in ("perm", "leaf_start", "leaf_count", "leaf_level", "leaf_prefix", "u_off", "u_idx"):
                assert np.array_equal(G[k], getattr(To2, k)), (flag, step, k)
            out.append(G)
            px, py, pz, qx, qy, qz = (a[To2.perm] for a in (px, py, pz, qx, qy, qz))
            To = To2
        res[flag] = (out, t.counters())
        t.close()
    # a key is captured on its second use (steps 0, 1 launch directly; 2..6 replay or capture + replay)
    assert res["1"][1]["graph_launches"] >= 5 and res["0"][1]["graph_launches"] == 0
    for step, (a, b) in enumerate(zip(res["1"][0], res["0"][0])):
        for k in a:
            assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), (step, k)


def _edits_for(t, rng, frac=0.1):
    """A seeded set of FineGrainedOptimize edits on the handle's current nodes:
    Collapse on some parents, PushDown on some leaves (incl. a level-21 cap case)."""
    nd = t.nodes()
    lev, pre, nch = nd["level"], nd["prefix"], nd["nchild"]
    pick = rng.random(lev.shape[0]) < frac
    return [(int(l), int(p), 1 if c > 0 else 2) for l, p, c, k in zip(lev, pre, nch, pick) if k]


def test_direct_keep_and_edits_match_level_loop(monkeypatch):
    """afmm_tree_rebuild (KEEP structure, or Enforce_S, with FineGrainedOptimize's
    Collapse / PushDown edits) through the direct construction -- per-body leaf level
    by bisection over the previous parents, edits applied along the path -- equals the
    level loop (AFMM_TREE_LEVELS=1) tree and node arrays, with and without CUDA graph
    replay, and the oracle's rebuild."""
    afmm = _afmm()
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(30000, 8)
    dom = synth.c5_domain(x, y, z)
    n = x.shape[0]
    plan = [(2, 0.0), (2, 0.0), (2, 0.1), (1, 0.05), (2, 0.0), (1, 0.0), (2, 0.2), (2, 0.2), (1, 0.1)]
    res = {}
    for levels, graph in (("0", "1"), ("0", "0"), ("1", "0")):
        monkeypatch.setenv("AFMM_TREE_LEVELS", levels)
        monkeypatch.setenv("AFMM_TREE_GRAPH", graph)
        rng = np.random.default_rng(11)
        t = afmm.GpuTree(0)
        bufs = [torch.empty((3, n), device="cuda") for _ in range(2)]
        S = 20
        t.build(_dev(x), _dev(y), _dev(z), S, domain=dom)
        To = oracle.Tree(x, y, z, S, domain=dom, ulist=False)
        px, py, pz, qx, qy, qz = (a[To.perm] for a in (x, y, z, vx, vy, vz))
        out = []
        for step, (mode, frac) in enumerate(plan):
            px, py, pz = oracle.drift(px, py, pz, qx, qy, qz, 0.2)
            ed = _edits_for(t, rng, frac) if frac > 0 else []
            b = bufs[step % 2]
            b.copy_(torch.from_numpy(np.stack([px, py, pz])))
            t.rebuild(b[0], b[1], b[2], S, mode=mode, edits=ed)
            G = _tree_and_nodes(t, n)
            To2 = To.rebuild(px, py, pz, S=S, mode=mode, edits=ed, ulist=False)
            for k in ("perm", "leaf_start", "leaf_count", "leaf_level", "leaf_prefix"):
                assert np.array_equal(G[k], getattr(To2, k)), (levels, graph, step, k)
            out.append(G)
            px, py, pz, qx, qy, qz = (a[To2.perm] for a in (px, py, pz, qx, qy, qz))
            To = To2
        res[levels + graph] = out
        t.close()
    for other in ("00", "10"):
        for step, (a, b) in enumerate(zip(res["01"], res[other])):
            for k in a:
                assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), (other, step, k)


@pytest.mark.parametrize("S,fallback", [(600, False), (3000, False), (20000, True)])
def test_large_buckets_cta_sort(S, fallback):
    """Rebuilds whose previous leaves hold more than the warp sort's 512 keys: buckets
    of up to 8192 keys are sorted by one CTA each in shared memory (no full-sort
    fallback), larger ones fall back to the full sort -- the tree bit-exact with the
    oracle's Enforce_S chain either way."""
    afmm = _afmm()
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(60000, 4)
    dom = synth.c5_domain(x, y, z)
    n = x.shape[0]
    t = afmm.GpuTree(0)
    t.build(_dev(x), _dev(y), _dev(z), S, domain=dom)
    To = oracle.Tree(x, y, z, S, domain=dom, ulist=False)
    assert To.leaf_count.max() > 512
    px, py, pz, qx, qy, qz = (a[To.perm] for a in (x, y, z, vx, vy, vz))
    for step in range(3):
        px, py, pz = oracle.drift(px, py, pz, qx, qy, qz, 0.2)
        t.enforce(_dev(px), _dev(py), _dev(pz), S)
        To2 = To.enforce(px, py, pz, S, ulist=False)
        G = t.copy_out(n)
        for k in ("perm", "leaf_start", "leaf_count", "leaf_level", "leaf_prefix"):
            assert np.array_equal(G[k], getattr(To2, k)), (S, step, k)
        px, py, pz, qx, qy, qz = (a[To2.perm] for a in (px, py, pz, qx, qy, qz))
        To = To2
    assert (t.counters()["sort_fallbacks"] > 0) == fallback
    t.close()


def test_randomised_builds_and_enforce_chains_bit_exact():
    """30 seeded random cases: n in [1, 30000], S in [1, 2100] (around the direct
    construction's tile and window limits: S = 2048 is its largest, 2049+ takes the
    level loop), uniform / Plummer / colliding / clustered duplicates, fresh builds
    and short Enforce_S chains with a changing S on one handle -- every tree and
    U-list bit-exact with the oracle."""
    afmm = _afmm()
    rng = np.random.default_rng(2026)
    dists = ("uniform", "plummer", "colliding")
    t = afmm.GpuTree(0)
    for case in range(30):
        n = int(rng.choice([1, 2, 3, 17, 63, 64, 65, 1000, 4096, 9999, 30000]))
        S = int(rng.choice([1, 2, 7, 31, 32, 33, 64, 100, 255, 1024, 2047, 2048, 2049, 2100]))
        x, y, z, m = synth.make(dists[case % 3], n, 100 + case)
        if case % 5 == 4:                                    # clustered duplicates
            idx = rng.integers(0, max(1, n // 7), n)
            x, y, z = x[idx], y[idx], z[idx]
        dom = (np.array([-16.0, -16.0, -16.0]), 5)
        t.build(_dev(x), _dev(y), _dev(z), S, domain=dom)
        To = oracle.Tree(x, y, z, S, domain=dom)
        assert_same_tree(t.copy_out(n), To)
        px, py, pz = x[To.perm], y[To.perm], z[To.perm]
        for step in range(2):
            S2 = max(1, int(S * rng.choice([0.5, 1.0, 1.5])))
            d = rng.standard_normal((3, n)).astype(np.float32) * np.float32(0.01)
            px, py, pz = (px + d[0]).astype(np.float32), (py + d[1]).astype(np.float32), (pz + d[2]).astype(np.float32)
            t.enforce(_dev(px), _dev(py), _dev(pz), S2)
            To2 = To.enforce(px, py, pz, S2)
            G = t.copy_out(n)
            for k in ("perm", "leaf_start", "leaf_count", "leaf_level", "leaf_prefix", "u_off", "u_idx"):
                assert np.array_equal(G[k], getattr(To2, k)), (case, n, S, S2, step, k)
            px, py, pz = px[To2.perm], py[To2.perm], pz[To2.perm]
            To = To2
    t.close()
