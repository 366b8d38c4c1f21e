"""Row f4: the regularized-Stokeslet pair law on the GPU (same pipeline,
Stokeslet policy) vs the fp64 oracle (reading R26)."""
import numpy as np
import pytest

import oracle
import synth
from tests import _tol

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _run(xs, ys, zs, fx, fy, fz, T, eps2, mu=1.0, world=1, slice_world=0):
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    n = xs.shape[0]
    out = torch.full((4, n), float("nan"), device="cuda")
    dev = [torch.from_numpy(np.ascontiguousarray(a, np.float32)).cuda() for a in (xs, ys, zs, fx, fy, fz)]
    for r in range(world):
        h = afmm.P2P(rank=r, world=world, eps2=eps2, law=afmm.LAW_STOKESLET, mu=mu, slice_world=slice_world)
        h.set_bodies_stokeslet(*dev)
        h.set_tree(T.leaf_start, T.leaf_count, T.u_off, T.u_idx)
        h.eval(out[0], out[1], out[2], out[3])
        h.close()
    torch.cuda.synchronize()
    return out.cpu().numpy()


@pytest.mark.parametrize("n,S,eps2,mu", [(5000, 64, 1e-4, 1.0), (200000, 128, 1e-6, 0.5), (3000, 1, 1e-3, 2.0)])
def test_stokeslet_parity(n, S, eps2, mu):
    x, y, z, fx, fy, fz = synth.uniform_with_forces(n, 11)
    T = oracle.Tree(x, y, z, S)
    xs, ys, zs, gx, gy, gz = T.sorted_bodies(x, y, z, fx, fy, fz)
    got = _run(xs, ys, zs, gx, gy, gz, T, eps2, mu)
    tg = None
    if n > 50000:
        tg = np.sort(np.random.default_rng(1).choice(T.L, 800, replace=False)).astype(np.int32)
    ref = oracle.stokeslet(xs, ys, zs, gx, gy, gz, T.leaf_start, T.leaf_count, T.u_off, T.u_idx, mu, eps2,
                           targets=tg, with_scale=True)
    sel = np.ones(n, bool) if tg is None else np.isfinite(ref[0])
    _tol.check_vec([g[sel] for g in got[:3]], [r[sel] for r in ref[:3]], ref[3][sel])
    assert (got[3] == 0).all()


def test_stokeslet_self_term_and_world_invariance():
    x = np.array([0.25], np.float32)
    f = [np.array([v], np.float32) for v in (1.0, -2.0, 0.5)]
    T = oracle.Tree(x, x, x, 4)
    got = _run(x, x, x, *f, T, 1e-4, 1.0)
    for c in range(3):
        assert got[c][0] == pytest.approx(float(f[c][0]) / (4 * np.pi * 1e-2), rel=1e-6)
    xx, yy, zz, fx, fy, fz = synth.uniform_with_forces(40000, 5)
    T = oracle.Tree(xx, yy, zz, 48)
    s = T.sorted_bodies(xx, yy, zz, fx, fy, fz)
    a = _run(*s, T, 1e-5, slice_world=3)
    b = _run(*s, T, 1e-5, world=3)
    assert np.array_equal(a, b)


def test_law_mismatch_is_einval():
    import paper_conf_ipps_overmanpmm13_b200 as afmm
    h = afmm.P2P(law=afmm.LAW_STOKESLET)
    v = torch.rand(8, device="cuda")
    with pytest.raises(afmm.AfmmError) as e:
        h.set_bodies(v, v, v, v)
    assert e.value.status == afmm.AFMM_EINVAL
    h.close()
    g = afmm.P2P()
    with pytest.raises(afmm.AfmmError) as e:
        g.set_bodies_stokeslet(v, v, v, v, v, v)
    assert e.value.status == afmm.AFMM_EINVAL
    g.close()
    with pytest.raises(afmm.AfmmError):
        afmm.P2P(law=7)
    with pytest.raises(afmm.AfmmError):
        afmm.P2P(law=afmm.LAW_STOKESLET, mu=0.0)
