"""C5 dynamic workload on the GPU vs the oracle:
leapfrog kernels (1 ulp), Enforce_S trees bit-exact at every step of a
trajectory, and per-step P2P parity on the GPU's own positions (trajectories
are chaotic, so parity is per step, not per trajectory -- SURVEY S8(d))."""
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


def _ulp_close(a, b, ulps=1):
    a = np.asarray(a, np.float32)
    b = np.asarray(b, np.float32)
    ia = a.view(np.int32).astype(np.int64)
    ib = b.view(np.int32).astype(np.int64)
    ia = np.where(ia < 0, -(ia & 0x7FFFFFFF), ia)
    ib = np.where(ib < 0, -(ib & 0x7FFFFFFF), ib)
    return np.abs(ia - ib).max() <= ulps


def test_leapfrog_kernels_vs_oracle():
    afmm = _afmm()
    rng = np.random.default_rng(2)
    n = 100003
    v = [rng.standard_normal(n).astype(np.float32) for _ in range(3)]
    a = [rng.standard_normal(n).astype(np.float32) * 10 for _ in range(3)]
    x = [rng.random(n).astype(np.float32) * 20 - 10 for _ in range(3)]
    h = np.float32(0.025)
    dv = [torch.from_numpy(t).cuda() for t in v]
    da = [torch.from_numpy(t).cuda() for t in a]
    dx = [torch.from_numpy(t).cuda() for t in x]
    afmm.kick(*dv, *da, h)
    afmm.drift(*dx, *dv, np.float32(0.05))
    torch.cuda.synchronize()
    rv = oracle.kick(*v, *a, float(h))
    rx = oracle.drift(*x, *rv, float(np.float32(0.05)))
    for g, r in zip(dv, rv):
        assert _ulp_close(g.cpu().numpy(), r)
    for g, r in zip(dx, rx):
        assert _ulp_close(g.cpu().numpy(), r)
    # the fused kick + drift (afmm_kick_drift, used by the C5 loop) is bit-identical to the two kernels
    fv = [torch.from_numpy(t).cuda() for t in v]
    fx = [torch.from_numpy(t).cuda() for t in x]
    afmm.kick_drift(*fx, *fv, *da, h, np.float32(0.05))
    torch.cuda.synchronize()
    for f, g in zip(fv + fx, dv + dx):
        assert torch.equal(f, g)


def test_gpu_enforce_bit_exact_along_trajectory():
    afmm = _afmm()
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(60000, 5)
    dom = synth.c5_domain(x, y, z)
    S = 32
    t = afmm.GpuTree(0)
    t.build(*[torch.from_numpy(a).cuda() for a in (x, y, z)], S, domain=dom)
    To = oracle.Tree(x, y, z, S, domain=dom)
    G = t.copy_out(60000)
    assert np.array_equal(G["perm"], To.perm) and np.array_equal(G["u_idx"], To.u_idx)
    px, py, pz, qx, qy, qz = (a[To.perm] for a in (x, y, z, vx, vy, vz))
    changed_structure = 0
    for step in range(8):
        px, py, pz = oracle.drift(px, py, pz, qx, qy, qz, 0.5)
        t.enforce(*[torch.from_numpy(a).cuda() for a in (px, py, pz)], S)
        To2 = To.enforce(px, py, pz)
        G = t.copy_out(60000)
        for k in ("perm", "leaf_start", "leaf_count", "leaf_level", "leaf_prefix", "u_off", "u_idx"):
            assert np.array_equal(G[k], getattr(To2, k)), (step, k)
        fresh = oracle.Tree(px, py, pz, S, domain=dom, ulist=False)
        changed_structure += int(fresh.L != To2.L)            # hysteresis visible vs a fresh build
        px, py, pz, qx, qy, qz = (a[To2.perm] for a in (px, py, pz, qx, qy, qz))
        To = To2
    assert changed_structure > 0
    t.close()


def test_c5_timeloop_per_step_parity():
    """A short C5 run (64 Ki colliding bodies, S = 64, dt = 0.05, eps2 = 1e-4):
    every Enforce_S tree bit-exact vs the oracle chain on the GPU's positions,
    P2P within R16 on sampled leaves at the first and last steps."""
    from paper_conf_ipps_overmanpmm13_b200.timeloop import TimeLoop
    n, S, eps2, dt = 1 << 16, 64, 1e-4, 0.05
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(n, 5)
    dom = synth.c5_domain(x, y, z)
    oracle_tree = [oracle.Tree(x, y, z, S, domain=dom)]
    loop = TimeLoop(x, y, z, m, vx, vy, vz, S, eps2, dt, dom)
    assert np.array_equal(loop.T["u_idx"], oracle_tree[0].u_idx)
    checks = {"trees": 0, "p2p": 0}

    def pre(px, py, pz):
        oracle_tree[0] = oracle_tree[0].enforce(px, py, pz)

    def post(lp):
        To = oracle_tree[0]
        for k in ("leaf_start", "leaf_count", "u_off", "u_idx"):
            assert np.array_equal(lp.T[k], getattr(To, k)), k
        checks["trees"] += 1
        if lp.step_no in (1, 12):
            s = lp.state.cpu().numpy()
            acc = lp.acc.cpu().numpy()
            rng = np.random.default_rng(lp.step_no)
            tg = np.sort(rng.choice(To.L, size=min(600, To.L), replace=False)).astype(np.int32)
            ref = oracle.p2p(s[0], s[1], s[2], s[3], To.leaf_start, To.leaf_count, To.u_off, To.u_idx,
                             1.0, eps2, targets=tg, with_scale=True)
            sel = np.zeros(n, bool)
            for t in tg:
                sel[To.leaf_start[t]:To.leaf_start[t] + To.leaf_count[t]] = True
            got = [acc[3][sel], acc[0][sel], acc[1][sel], acc[2][sel]]
            _tol.check(got, [r[sel] for r in ref[:4]], ref[4][sel])
            checks["p2p"] += 1

    for _ in range(12):
        rec = loop.step({"pre_enforce": pre, "post_eval": post})
        assert rec["interactions"] > 0
    assert checks["trees"] == 12 and checks["p2p"] == 2
    # momentum of the near-field system (symmetric U-lists) is conserved to fp32 round-off
    s = loop.state.cpu().numpy().astype(np.float64)
    p = (s[3][None, :] * s[4:7]).sum(1)
    p0 = (m.astype(float)[None, :] * np.stack([vx, vy, vz]).astype(float)).sum(1)
    assert np.abs(p - p0).max() < 1e-4
    loop.close()


def test_c5_async_steps_bit_identical():
    """TimeLoop.step(sync=False) (steps enqueued back to back, one synchronise in
    finish) gives a trajectory bit-identical to synchronised steps, and finish()
    fills every record's timings (the bench's C5 line runs this way)."""
    from paper_conf_ipps_overmanpmm13_b200.timeloop import TimeLoop
    n, S, eps2, dt = 1 << 16, 64, 1e-4, 0.05
    x, y, z, m, vx, vy, vz = synth.colliding_with_velocities(n, 8)
    dom = synth.c5_domain(x, y, z)
    a = TimeLoop(x, y, z, m, vx, vy, vz, S, eps2, dt, dom)
    for _ in range(8):
        a.step()
    sa = a.state.cpu().numpy().copy()
    a.close()
    b = TimeLoop(x, y, z, m, vx, vy, vz, S, eps2, dt, dom)
    recs = [b.step(sync=False) for _ in range(8)]
    b.finish(recs)
    sb = b.state.cpu().numpy().copy()
    b.close()
    assert np.array_equal(sa, sb)
    for r in recs:
        assert r["kernel_ms"] > 0 and r["enforce_ms"] > 0 and r["interactions"] > 0 and "_events" not in r
