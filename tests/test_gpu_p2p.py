"""GPU parity of the CUDA P2P path (through the C ABI) against the fp64 oracle.

Tolerance: DESIGN.md reading R16 (tests/_tol.py).  Integer tree inputs come
from the oracle here; tests/test_gpu_tree.py checks the GPU tree builder
bit-exactly against it and runs the full-size configs end to end."""
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


def gpu_eval(xs, ys, zs, ms, T, eps2, G=1.0, world=1, max_leaf=None, leaf_split=None, slice_world=0):
    """Run the library for every rank of `world` on this one GPU and merge the
    disjoint output slices (ranks write only their own bodies)."""
    afmm = _afmm()
    n = xs.shape[0]
    out = [torch.full((n,), float("nan"), device="cuda") for _ in range(4)]
    bodies = [_dev(v) for v in (xs, ys, zs, ms)]
    stats = []
    for r in range(world):
        h = afmm.P2P(device=0, rank=r, world=world, G=G, eps2=eps2, max_leaf=max_leaf, slice_world=slice_world)
        h.set_bodies(*bodies)
        if leaf_split is not None:
            h.set_partition(leaf_split)
        h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
        stats.append(h.eval(*out, stats=True))
        h.close()
    torch.cuda.synchronize()
    ax, ay, az, phi = (o.cpu().numpy() for o in out)
    return (phi, ax, ay, az), stats                 # the oracle's order


def _tree(x, y, z, S):
    T = oracle.Tree(x, y, z, S)
    return T, {"leaf_start": T.leaf_start, "leaf_count": T.leaf_count, "u_off": T.u_off,
               "u_idx": T.u_idx}


def _parity(x, y, z, m, S, eps2, G=1.0, targets=None, world=1):
    T, d = _tree(x, y, z, S)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    got, stats = gpu_eval(xs, ys, zs, ms, d, eps2, G, world=world)
    ref = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, G, eps2,
                     targets=targets, with_scale=True)
    sel = np.ones(xs.shape[0], bool)
    if targets is not None:
        sel[:] = False
        for t in targets:
            sel[T.leaf_start[t]:T.leaf_start[t] + T.leaf_count[t]] = True
    e = _tol.check([g[sel] for g in got], [r[sel] for r in ref[:4]], ref[4][sel])
    I = oracle.interactions(T.leaf_count, T.u_off, T.u_idx)
    assert sum(s["interactions_rank"] for s in stats) == int(I.sum())
    assert stats[0]["interactions_total"] == int(I.sum())
    return e, got, T


def test_c1_parity():
    x, y, z, m = synth.make("C1")
    e, _, _ = _parity(x, y, z, m, 64, 1e-6)
    assert e["phi_max_rel"] < 2e-6


@pytest.mark.parametrize("S", [32, 128, 512])
def test_c2_plummer_parity_full(S):
    """C2 (1M Plummer) at three points of the S sweep, every body checked."""
    x, y, z, m = synth.make("C2")
    _parity(x, y, z, m, S, 1e-6)


def test_c3_colliding_parity_full():
    x, y, z, m = synth.make("C3")
    _parity(x, y, z, m, 128, 1e-6)


@pytest.mark.parametrize("dist,n,S,eps2", [("uniform", 20000, 1, 1e-6), ("uniform", 20000, 7, 0.0),
                                           ("plummer", 50000, 300, 1e-4), ("colliding", 30000, 33, 1e-6),
                                           ("plummer", 1000, 5000, 1e-6), ("plummer", 40000, 3000, 1e-6),
                                           ("uniform", 30000, 12000, 1e-6)])
def test_ragged_leaf_sizes(dist, n, S, eps2):
    """Leaves of every size 1..S (ragged tails of the lane mapping), eps2 = 0,
    one-leaf trees (N <= S), sources spanning several 1024-body stages, leaves
    far above 1024 bodies (the KEEP rule of the load balancer lets leaves grow)."""
    x, y, z, m = synth.make(dist, n, 17)
    _parity(x, y, z, m, S, eps2)


def test_single_body_and_two_bodies():
    afmm = _afmm()
    x = np.array([0.25], np.float32)
    T, d = _tree(x, x, x, 1)
    got, _ = gpu_eval(x, x, x, np.ones(1, np.float32), d, 0.0)
    assert all(g[0] == 0.0 for g in got)          # self entry only, n_t = 1 -> exactly 0
    x = np.array([0.25, 0.75], np.float32)
    y = np.array([0.5, 0.125], np.float32)
    z = np.array([0.0, 0.5], np.float32)
    m = np.array([0.5, 0.25], np.float32)
    for S in (1, 2):
        T, d = _tree(x, y, z, S)
        xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
        got, _ = gpu_eval(xs, ys, zs, ms, d, 1e-2, G=2.0)
        for i in range(2):
            j = 1 - i
            dd = np.array([xs[j] - xs[i], ys[j] - ys[i], zs[j] - zs[i]], float)
            r2 = dd @ dd + 1e-2
            assert got[0][i] == pytest.approx(-2.0 * ms[j] / np.sqrt(r2), rel=1e-6)
            assert np.allclose([got[1][i], got[2][i], got[3][i]], 2.0 * ms[j] * dd / r2 ** 1.5, rtol=1e-6)


def test_big_leaves_target_chunking():
    """Level-21 leaves larger than 512 targets (split into target chunks) and
    larger than one 1024-body stage."""
    rng = np.random.default_rng(3)
    base = np.array([0.5, 0.5, 0.5])
    cl = base + rng.random((1000, 3)) * 1e-7             # one quantisation cell
    far = rng.random((3000, 3))
    P = np.concatenate([cl, far, [[0, 0, 0], [0.999, 0.999, 0.999]]]).astype(np.float32)
    m = np.full(P.shape[0], 1.0 / P.shape[0], np.float32)
    x, y, z = P[:, 0].copy(), P[:, 1].copy(), P[:, 2].copy()
    T = oracle.Tree(x, y, z, 16)
    assert T.leaf_count.max() >= 900 and T.leaf_level[T.leaf_count.argmax()] == 21
    e, _, _ = _parity(x, y, z, m, 16, 1e-12)


def test_deterministic_and_world_invariant():
    """Bit-identical results across repeated evals and world sizes 1/2/3/8 for
    one task slicing (slice_world = 8); the production slicing (slice_world =
    world) agrees within R16."""
    x, y, z, m = synth.make("plummer", 200000, 9)
    T, d = _tree(x, y, z, 64)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    ref, _ = gpu_eval(xs, ys, zs, ms, d, 1e-6, slice_world=8)
    again, _ = gpu_eval(xs, ys, zs, ms, d, 1e-6, slice_world=8)
    for a, b in zip(ref, again):
        assert np.array_equal(a, b)
    oref = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-6, with_scale=True)
    for W in (2, 3, 8):
        prod, _ = gpu_eval(xs, ys, zs, ms, d, 1e-6, world=W)
        _tol.check(list(prod), list(oref[:4]), oref[4])
        got, stats = gpu_eval(xs, ys, zs, ms, d, 1e-6, world=W, slice_world=8)
        for a, b in zip(ref, got):
            assert np.array_equal(a, b)
        # ranks own disjoint contiguous slices covering every body
        lo = [s["body_lo"] for s in stats]
        hi = [s["body_hi"] for s in stats]
        assert lo[0] == 0 and hi[-1] == xs.shape[0] and all(hi[i] == lo[i + 1] for i in range(W - 1))


def test_mass_scaling_bit_exact():
    x, y, z, m = synth.make("plummer", 50000, 4)
    T, d = _tree(x, y, z, 48)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    a, _ = gpu_eval(xs, ys, zs, ms, d, 1e-6)
    b, _ = gpu_eval(xs, ys, zs, (ms * np.float32(8)).astype(np.float32), d, 1e-6)
    for u, v in zip(a, b):
        assert np.array_equal(v, u * np.float32(8))


def test_momentum_conservation():
    """Newton's third law on the GPU result (symmetric U): |sum m a| small vs sum m A."""
    x, y, z, m = synth.make("plummer", 100000, 6)
    T, d = _tree(x, y, z, 64)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    got, _ = gpu_eval(xs, ys, zs, ms, d, 1e-6)
    ref = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-6,
                     with_scale=True)
    mm = ms.astype(np.float64)
    scale = (mm * ref[4]).sum()
    for c in range(3):
        assert abs((mm * got[1 + c].astype(np.float64)).sum()) <= 1e-6 * scale


def test_host_pointer_api_matches_device_api():
    afmm = _afmm()
    x, y, z, m = synth.make("C1")
    T, d = _tree(x, y, z, 64)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    ref, _ = gpu_eval(xs, ys, zs, ms, d, 1e-6)
    h = afmm.P2P(eps2=1e-6)
    h.set_bodies(xs, ys, zs, ms)                     # numpy -> afmm_p2p_set_bodies_host
    h.set_tree(d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
    out = [np.zeros(xs.shape[0], np.float32) for _ in range(4)]
    st = h.eval(*out)                                # numpy -> afmm_p2p_eval_host (blocking)
    for a, b in zip(ref, [out[3], out[0], out[1], out[2]]):
        assert np.array_equal(a, b)
    assert st["n_launches"] == 1 and st["kernel_ms"] > 0
    h.close()


def test_error_statuses():
    afmm = _afmm()
    with pytest.raises(afmm.AfmmError) as e:
        afmm.P2P(max_leaf=afmm.MAX_LEAF + 1)
    assert e.value.status == afmm.AFMM_ENOTSUP
    for kw in ({"eps2": -1.0}, {"G": float("inf")}, {"world": 0}, {"rank": 2, "world": 2}):
        with pytest.raises(afmm.AfmmError) as e:
            afmm.P2P(**kw)
        assert e.value.status == afmm.AFMM_EINVAL
    h = afmm.P2P(max_leaf=64)
    out = [torch.zeros(8, device="cuda") for _ in range(4)]
    with pytest.raises(afmm.AfmmError) as e:
        h.eval(*out)
    assert e.value.status == afmm.AFMM_ESTATE
    with pytest.raises(afmm.AfmmError) as e:
        h.set_tree([0], [8], [0, 1], [0])
    assert e.value.status == afmm.AFMM_ESTATE
    xs = torch.rand(8, device="cuda")
    h.set_bodies(xs, xs, xs, xs)
    bad = [
        ([0, 4], [4, 3], [0, 1, 2], [0, 1]),          # leaves do not cover n
        ([0, 5], [4, 4], [0, 1, 2], [0, 1]),          # gap between leaves
        ([0, 4], [4, 4], [0, 2, 3], [1, 0, 1]),       # row not ascending
        ([0, 4], [4, 4], [0, 1, 3], [0, 1, 1]),       # duplicate entry in a row
        ([0, 4], [4, 4], [0, 1, 2], [0, 2]),          # index out of range
        ([0, 4], [4, 4], [1, 1, 2], [0, 1]),          # u_off[0] != 0
        ([0, 4], [4, 4], [0, 2, 1], [0, 1]),          # u_off not monotone
    ]
    for ls, lc, uo, ui in bad:
        with pytest.raises(afmm.AfmmError) as e:
            h.set_tree(ls, lc, uo, ui)
        assert e.value.status == afmm.AFMM_EINVAL
    h2 = afmm.P2P(max_leaf=4)
    h2.set_bodies(xs, xs, xs, xs)
    with pytest.raises(afmm.AfmmError) as e:
        h2.set_tree([0, 2], [2, 6], [0, 1, 2], [0, 1])          # 6 > max_leaf
    assert e.value.status == afmm.AFMM_EINVAL
    h2.close()
    # the handle stays usable after EINVAL
    h.set_tree([0, 4], [4, 4], [0, 2, 4], [0, 1, 0, 1])
    h.eval(*out, stats=True)
    with pytest.raises(afmm.AfmmError) as e:
        h.set_bodies(None, None, None, None, n=0)
    assert e.value.status == afmm.AFMM_EINVAL
    h.close()


def test_rebalance_keeps_results_and_valid_split():
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", 100000, 8)
    T, d = _tree(x, y, z, 64)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    ref, _ = gpu_eval(xs, ys, zs, ms, d, 1e-6, slice_world=4)
    W = 4
    hs = [afmm.P2P(rank=r, world=W, eps2=1e-6) for r in range(W)]
    bodies = [_dev(v) for v in (xs, ys, zs, ms)]
    for h in hs:
        h.set_bodies(*bodies)
        h.set_tree(d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
    fake_ms = np.array([1.0, 2.0, 1.0, 1.0])              # rank 1 "slow"
    changed = [h.rebalance(fake_ms, 0.02) for h in hs]
    assert len(set(changed)) == 1 and changed[0]
    splits = [h.get_partition()[0] for h in hs]
    assert all(np.array_equal(splits[0], s) for s in splits)
    sp = splits[0]
    assert sp[0] == 0 and sp[-1] == T.L and (np.diff(sp) >= 0).all()
    out = [torch.full((xs.shape[0],), float("nan"), device="cuda") for _ in range(4)]
    for h in hs:
        h.eval(*out)
    torch.cuda.synchronize()
    for a, b in zip(ref, [out[3], out[0], out[1], out[2]]):
        assert np.array_equal(a, b.cpu().numpy())
    for h in hs:
        h.close()


def test_fp32_peak_sane():
    afmm = _afmm()
    p = afmm.fp32_peak(0)
    assert 30 < p["ffma_tflops"] < 90 and 20 < p["ffma2_tflops"] < 180


@pytest.mark.parametrize("world,coef", [(1, None), (3, None), (4, [1.0, 1.0, 2.0, 1.5, 1.0, 1.0, 1.0, 1.0])])
def test_set_tree_device_matches_host_ingest(world, coef, monkeypatch):
    """afmm_p2p_set_tree_device (kernels) == the host work-list builder
    (AFMM_HOST_INGEST=1) == afmm_p2p_set_tree on host arrays (copied, then the
    device ingest): same partition, stats and bit-identical outputs."""
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", 150000, 12)
    n = x.shape[0]
    tree = afmm.GpuTree(0)
    X, Y, Z, M = (torch.from_numpy(v).cuda() for v in (x, y, z, m))
    info = tree.build(X, Y, Z, 48)
    T = tree.copy_out(n)
    d = tree.device_arrays()
    bod = torch.empty((4, n), device="cuda")
    for a, src in enumerate((X, Y, Z, M)):
        tree.gather(src, bod[a])
    outs, worklists = [], []
    for mode in ("host", "device", "host-arrays"):
        monkeypatch.setenv("AFMM_HOST_INGEST", "1" if mode == "host" else "0")
        out = torch.full((4, n), float("nan"), device="cuda")
        splits, stats, wls = [], [], []
        for r in range(world):
            h = afmm.P2P(rank=r, world=world, eps2=1e-6)
            h.set_bodies(bod[0], bod[1], bod[2], bod[3])
            if coef is not None:
                h.set_cost_coef(coef)
            if mode != "device":
                h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
            else:
                h.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
            stats.append(h.eval(out[0], out[1], out[2], out[3], stats=True))
            splits.append(h.get_partition())
            wls.append(h.worklist())
            h.close()
        torch.cuda.synchronize()
        outs.append((out.cpu().numpy(), splits, stats))
        worklists.append(wls)
    (oh, sh, th), (od, sd, td), (oa, sa, ta) = outs
    if coef is None:                            # the same work list, task for task (dispatch order included)
        for (tw, sw), (tdv, sdv), (ta_, sa_) in zip(*worklists):
            assert tw.shape[0] > 0
            assert np.array_equal(tw, tdv) and np.array_equal(sw, sdv)
            assert np.array_equal(ta_, tdv) and np.array_equal(sa_, sdv)
            cost = -(-np.maximum(tdv[:, 6], 1) // (32 // (-(-tdv[:, 1] // 4))))
            assert (np.diff(cost) <= 0).all()     # largest modelled cost first
    assert np.array_equal(oh, od) and np.isfinite(od).all()
    assert np.array_equal(oa, od)
    for a, b in zip(sa, sd):
        assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    for a, b in zip(ta, td):
        for k in ("interactions_total", "interactions_rank", "bucket_interactions", "n_work_items", "leaf_lo",
                  "leaf_hi", "body_lo", "body_hi"):
            assert a[k] == b[k], k
    for a, b in zip(sh, sd):
        if coef is None:
            assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
        else:                                   # fp64 prefix sums of the weights may tie-break differently
            assert np.abs(a[0] - b[0]).max() <= 1
    for a, b in zip(th, td):
        assert a["interactions_total"] == b["interactions_total"]
        if coef is None:
            assert a["interactions_rank"] == b["interactions_rank"]
            assert a["bucket_interactions"] == b["bucket_interactions"]
            assert a["n_work_items"] == b["n_work_items"]
    tree.close()


def test_set_tree_device_rejects_invalid_tree():
    afmm = _afmm()
    h = afmm.P2P(max_leaf=64)
    xs = torch.rand(8, device="cuda")
    h.set_bodies(xs, xs, xs, xs)
    dev = lambda a, dt: torch.tensor(a, dtype=dt, device="cuda")  # noqa: E731
    bad = [([0, 4], [4, 3], [0, 1, 2], [0, 1]), ([0, 4], [4, 4], [0, 2, 3], [1, 0, 1]),
           ([0, 4], [4, 4], [0, 1, 2], [0, 2]), ([0, 4], [4, 4], [1, 1, 2], [0, 1])]
    for ls, lc, uo, ui in bad:
        with pytest.raises(afmm.AfmmError) as e:
            h.set_tree_device(2, dev(ls, torch.int32), dev(lc, torch.int32), dev(uo, torch.int64),
                              dev(ui, torch.int32))
        assert e.value.status == afmm.AFMM_EINVAL
    h.set_tree_device(2, dev([0, 4], torch.int32), dev([4, 4], torch.int32), dev([0, 2, 4], torch.int64),
                      dev([0, 1, 0, 1], torch.int32))
    out = [torch.zeros(8, device="cuda") for _ in range(4)]
    h.eval(*out, stats=True)
    assert h.rebalance([1.0], 0.02) is False       # the handle keeps its own copy of the tree
    h.close()


@pytest.mark.parametrize("world,pieces,ingest,zc", [(1, 1, "host", "1"), (1, 8, "host", "0"), (1, 64, "device", "0"),
                                                    (1, 8, "device", "1"), (2, 5, "host", "0"), (2, 5, "host", "1"),
                                                    (3, 8, "device", "1")])
def test_eval_host_pipelined_bit_identical(world, pieces, ingest, zc, monkeypatch):
    """afmm_p2p_eval_host_pipelined (H2D / kernel pieces / D2H overlapped;
    zc = "1": zero-copy, the kernels read and write the pinned host arrays) ==
    afmm_p2p_eval on device buffers, bit for bit, on every rank's slice; the
    handle's bodies afterwards are the host ones (a plain eval agrees too).
    Unequal masses: both take the general pair loop."""
    monkeypatch.setenv("AFMM_E2E_ZEROCOPY", zc)
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", 200000, 21)
    m = (m * np.random.default_rng(3).uniform(0.5, 1.5, m.shape[0])).astype(np.float32)
    n = x.shape[0]
    tree = afmm.GpuTree(0)
    X, Y, Z, M = (torch.from_numpy(v).cuda() for v in (x, y, z, m))
    info = tree.build(X, Y, Z, 64)
    T = tree.copy_out(n)
    d = tree.device_arrays()
    bod = torch.empty((4, n), device="cuda")
    for a, src in enumerate((X, Y, Z, M)):
        tree.gather(src, bod[a])
    hb = [bod[a].cpu().pin_memory() for a in range(4)]
    ref = torch.full((4, n), float("nan"), device="cuda")
    got = [torch.full((n,), float("nan")).pin_memory() for _ in range(4)]
    again = torch.full((4, n), float("nan"), device="cuda")
    for r in range(world):
        h = afmm.P2P(rank=r, world=world, eps2=1e-6)
        h.set_bodies(bod[0], bod[1], bod[2], bod[3])
        if ingest == "host":
            h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
        else:
            h.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
        h.eval(ref[0], ref[1], ref[2], ref[3])
        h.set_bodies(*[torch.zeros(n, device="cuda") for _ in range(4)])   # stale device bodies
        for _ in range(2):                                                  # plan reused on the 2nd call
            st = h.eval_host_pipelined(*hb, *got, pieces=pieces)
        assert st["n_launches"] <= pieces and st["n_launches"] >= 1
        assert st["zero_copy"] == int(zc)
        assert st["input_graph"] == int(zc)            # zero-copy inputs: the chain replays from a graph
        h.eval(again[0], again[1], again[2], again[3])
        h.close()
    torch.cuda.synchronize()
    r_ = ref.cpu().numpy()
    assert np.isfinite(r_).all()
    for a in range(4):
        assert np.array_equal(got[a].numpy(), r_[a])
    assert np.array_equal(again.cpu().numpy(), r_)
    tree.close()


@pytest.mark.parametrize("offset,n,graph", [(0, 199997, "1"), (1, 200000, "1"), (3, 99999, "1"), (0, 200000, "0"),
                                           (1, 99999, "0")])
def test_eval_host_pipelined_zero_copy_ragged_and_misaligned(offset, n, graph, monkeypatch):
    """Zero-copy streamed inputs with chunk lengths not a multiple of 4 and host
    arrays that are not 16-byte aligned (views at an element offset into pinned
    buffers): the pack kernel's float4 path, its scalar tail and its scalar
    fallback all give results bit-identical to afmm_p2p_eval on device buffers,
    with the input chain replayed from its captured graph (graph = "1") or
    launched directly (AFMM_INPUT_GRAPH=0)."""
    monkeypatch.setenv("AFMM_E2E_ZEROCOPY", "1")
    monkeypatch.setenv("AFMM_INPUT_GRAPH", graph)
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", n, 24)
    tree = afmm.GpuTree(0)
    X, Y, Z, M = (torch.from_numpy(v).cuda() for v in (x, y, z, m))
    tree.build(X, Y, Z, 64)
    T = tree.copy_out(n)
    bod = torch.empty((4, n), device="cuda")
    for a, src in enumerate((X, Y, Z, M)):
        tree.gather(src, bod[a])
    hb = []
    for a in range(4):
        buf = torch.empty(n + offset).pin_memory()
        buf[offset:].copy_(bod[a].cpu())
        hb.append(buf[offset:])
    got = []
    for a in range(4):
        buf = torch.full((n + offset,), float("nan")).pin_memory()
        got.append(buf[offset:])
    ref = torch.full((4, n), float("nan"), device="cuda")
    h = afmm.P2P(eps2=1e-6)
    h.set_bodies(bod[0], bod[1], bod[2], bod[3])
    h.set_tree(T["leaf_start"], T["leaf_count"], T["u_off"], T["u_idx"])
    h.eval(ref[0], ref[1], ref[2], ref[3])
    h.set_bodies(*[torch.zeros(n, device="cuda") for _ in range(4)])   # stale device bodies
    st = h.eval_host_pipelined(*hb, *got, pieces=1)
    assert st["zero_copy"] == 1 and st["input_graph"] == int(graph)
    for a in range(4):
        assert np.array_equal(got[a].numpy(), ref[a].cpu().numpy())
    # a changed host array (new pointer) re-captures the input chain; same results
    hb[0] = hb[0].clone().pin_memory()
    for a in range(4):
        got[a].fill_(float("nan"))
    st = h.eval_host_pipelined(*hb, *got, pieces=1)
    assert st["input_graph"] == int(graph)
    h.close()
    tree.close()
    r_ = ref.cpu().numpy()
    assert np.isfinite(r_).all()
    for a in range(4):
        assert np.array_equal(got[a].numpy(), r_[a])


@pytest.mark.parametrize("zc", ["0", "1"])
def test_eval_host_pipelined_equal_masses(zc, monkeypatch):
    """Equal masses: the streamed chunks are flagged equal-mass, so
    eval_host_pipelined runs the equal-mass loop like eval: bit-identical to it,
    and both within R16 of the oracle.  One changed mass in the last chunk sends
    the tasks that reach it (only those) to the general loop: still within R16."""
    monkeypatch.setenv("AFMM_E2E_ZEROCOPY", zc)
    afmm = _afmm()
    x, y, z, m = synth.make("plummer", 60000, 22)
    T, d = _tree(x, y, z, 64)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    ref = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-6, with_scale=True)
    dev_out, _ = gpu_eval(xs, ys, zs, ms, d, 1e-6)
    h = afmm.P2P(eps2=1e-6)
    h.set_bodies(*[_dev(v) for v in (xs, ys, zs, ms)])
    h.set_tree(d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
    hb = [torch.from_numpy(np.ascontiguousarray(v, np.float32)).pin_memory() for v in (xs, ys, zs, ms)]
    got = [torch.empty(xs.shape[0]).pin_memory() for _ in range(4)]
    st = h.eval_host_pipelined(*hb, *got, pieces=3)
    assert st["zero_copy"] == int(zc)
    pipe = tuple(got[a].numpy().copy() for a in (3, 0, 1, 2))     # oracle order phi, ax, ay, az
    for a in range(4):
        assert np.array_equal(pipe[a], dev_out[a])
    _tol.check(list(pipe), list(ref[:4]), ref[4])
    _tol.check(list(dev_out), list(ref[:4]), ref[4])
    # perturb one mass in the last input chunk (x1.5): general loop for the tasks reaching it
    n = xs.shape[0]
    ms2 = ms.copy()
    ms2[n - 5] *= 1.5
    hb[3].copy_(torch.from_numpy(np.ascontiguousarray(ms2, np.float32)))
    ref2 = oracle.p2p(xs, ys, zs, ms2, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-6, with_scale=True)
    h.eval_host_pipelined(*hb, *got, pieces=3)
    h.close()
    pipe2 = (got[3].numpy(), got[0].numpy(), got[1].numpy(), got[2].numpy())
    _tol.check(list(pipe2), list(ref2[:4]), ref2[4])
    assert not np.array_equal(pipe2[0], pipe[0])


def test_eval_host_pipelined_errors():
    afmm = _afmm()
    h = afmm.P2P(eps2=1e-6)
    a = [np.zeros(10, np.float32) for _ in range(8)]
    with pytest.raises(afmm.AfmmError) as e:
        h.eval_host_pipelined(*a)
    assert e.value.status == afmm.AFMM_ESTATE
    x, y, z, m = synth.make("uniform", 1000, 3)
    T, dd = _tree(x, y, z, 32)
    h.set_bodies(*T.sorted_bodies(x, y, z, m))
    h.set_tree(dd["leaf_start"], dd["leaf_count"], dd["u_off"], dd["u_idx"])
    b = [np.zeros(1000, np.float32) for _ in range(8)]
    for p in (0, 65):
        with pytest.raises(afmm.AfmmError) as e:
            h.eval_host_pipelined(*b, pieces=p)
        assert e.value.status == afmm.AFMM_EINVAL
    with pytest.raises(afmm.AfmmError):
        h.eval_host_pipelined(*[np.zeros(999, np.float32) for _ in range(8)])
    h.close()
    s = afmm.P2P(law=afmm.LAW_STOKESLET)
    with pytest.raises(afmm.AfmmError) as e:
        s.eval_host_pipelined(*b)
    s.close()


def test_task_cap_splits_for_strong_scaling():
    """slice_world = 8 caps every task at I_total / 8 / (128 * warps * 3) warp
    iterations: more, smaller tasks than slice_world = 1, results within R16 of
    the oracle either way (a leaf's targets may be cut, its sums not)."""
    x, y, z, m = synth.make("plummer", 300000, 31)
    T, d = _tree(x, y, z, 128)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    ref = oracle.p2p(xs, ys, zs, ms, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-6, with_scale=True)
    items = {}
    for sw in (1, 8):
        got, stats = gpu_eval(xs, ys, zs, ms, d, 1e-6, slice_world=sw)
        _tol.check(list(got), list(ref[:4]), ref[4])
        items[sw] = stats[0]["n_work_items"]
    assert items[8] > items[1]


def test_unequal_masses_general_path_and_equal_mass_path():
    """The synthetic workloads have equal masses (R19), which the kernel detects
    (pack flag) and evaluates with the 12-op pair loop, applying G m once at the
    end.  Unequal masses take the general 13-op loop.  Both against the oracle
    (R16); equal masses scaled by 2^k scale the outputs bit-exactly on both."""
    x, y, z, m = synth.make("plummer", 120000, 41)
    T, d = _tree(x, y, z, 96)
    xs, ys, zs, ms = T.sorted_bodies(x, y, z, m)
    rng = np.random.default_rng(5)
    mu = (ms * rng.uniform(0.5, 1.5, ms.shape[0])).astype(np.float32)     # unequal
    for mm in (ms, mu):
        ref = oracle.p2p(xs, ys, zs, mm, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-6, with_scale=True)
        got, _ = gpu_eval(xs, ys, zs, mm, d, 1e-6)
        _tol.check(list(got), list(ref[:4]), ref[4])
    # one body's mass differs by one ulp: the general loop, within R16 of the oracle
    m1 = ms.copy()
    m1[777] = np.nextafter(m1[777], np.float32(1))
    ref1 = oracle.p2p(xs, ys, zs, m1, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, 1.0, 1e-6, with_scale=True)
    g_1, _ = gpu_eval(xs, ys, zs, m1, d, 1e-6)
    _tol.check(list(g_1), list(ref1[:4]), ref1[4])
    g_eq, _ = gpu_eval(xs, ys, zs, ms, d, 1e-6)
    assert not all(np.array_equal(a, b) for a, b in zip(g_eq, g_1))     # the two loops round differently
    g8, _ = gpu_eval(xs, ys, zs, (ms * 8).astype(np.float32), d, 1e-6)
    for a, b in zip(g_eq, g8):
        assert np.array_equal(a * 8, b)


def test_eval_host_pipelined_large_quadratic_chunks(monkeypatch):
    """Above 8 Mi bodies the streamed host-to-host evaluation cuts its input into
    one chunk per Mi bodies with quadratic boundaries n (k/K)^2 (afmm_p2p.cu
    chunk_bound): on 9 Mi Plummer bodies (K = 9, an odd n) its outputs are
    bit-identical to afmm_p2p_eval on device buffers, zero-copy in and out."""
    monkeypatch.setenv("AFMM_E2E_ZEROCOPY", "1")
    afmm = _afmm()
    n = 9 * (1 << 20) + 3
    x, y, z, m = synth.make("plummer", n, 29)
    tree = afmm.GpuTree(0)
    X, Y, Z, M = (torch.from_numpy(v).cuda() for v in (x, y, z, m))
    info = tree.build(X, Y, Z, 256)
    d = tree.device_arrays()
    bod = torch.empty((4, n), device="cuda")
    for a, src in enumerate((X, Y, Z, M)):
        tree.gather(src, bod[a])
    hb = [bod[a].cpu().pin_memory() for a in range(4)]
    got = [torch.full((n,), float("nan")).pin_memory() for _ in range(4)]
    ref = torch.full((4, n), float("nan"), device="cuda")
    h = afmm.P2P(eps2=1e-6)
    h.set_bodies(bod[0], bod[1], bod[2], bod[3])
    h.set_tree_device(info["n_leaves"], d["leaf_start"], d["leaf_count"], d["u_off"], d["u_idx"])
    h.eval(ref[0], ref[1], ref[2], ref[3])
    st = h.eval_host_pipelined(*hb, *got, pieces=1)
    assert st["zero_copy"] == 1
    r_ = ref.cpu().numpy()
    assert np.isfinite(r_).all()
    for a in range(4):
        assert np.array_equal(got[a].numpy(), r_[a])
    h.close()
    tree.close()


def test_randomised_parity():
    """24 seeded random cases against the fp64 oracle (reading R16): n in [2, 20000],
    S in [1, 300], uniform / Plummer / colliding positions, equal or random masses
    (the equal-mass and general pair loops), eps^2 in {0 (distinct points only),
    1e-8, 1e-6, 1e-3}, G != 1, worlds 1..3 merged -- plus the interaction count."""
    rng = np.random.default_rng(77)
    dists = ("uniform", "plummer", "colliding")
    for case in range(24):
        n = int(rng.choice([2, 5, 33, 500, 2048, 7777, 20000]))
        S = int(rng.choice([1, 3, 8, 17, 64, 128, 200, 300]))
        eps2 = float(rng.choice([0.0, 1e-8, 1e-6, 1e-3]))
        x, y, z, m = synth.make(dists[case % 3], n, 500 + case)
        if case % 2:
            m = rng.uniform(0.5, 2.0, n).astype(np.float32) / np.float32(n)
        if eps2 == 0.0:                                   # R21: coincident bodies need a softening
            keys = np.stack([x, y, z], 1)
            if np.unique(keys, axis=0).shape[0] < n:
                eps2 = 1e-8
        G = float(rng.choice([1.0, 0.5, 6.674e-11]))
        world = int(rng.choice([1, 2, 3]))
        _parity(x, y, z, m, S, eps2, G=G, world=world)
